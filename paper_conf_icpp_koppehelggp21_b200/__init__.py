"""B200-native CuART hot path: thin Python binding over the C ABI (include/cuart.h).

Argument marshalling only — every step of the path (build/flatten on the host in
C++, lookups and updates in the sm_100a kernels) runs inside ``libcuart.so``.
There is no Python or CPU fallback for the GPU calls: if the library or a GPU is
missing, the calls raise.

Names follow the C ABI: ``cuart_build``, ``cuart_lookup``, ``cuart_update``,
``cuart_destroy`` (plus ``*_host`` variants taking host buffers, introspection,
and the host-layout calls used by the CPU tests).  ``Index`` wraps a handle.
"""
from __future__ import annotations

from ._binding import (  # noqa: F401
    CUART_MISS, CUART_MAX_KEY, CuartError, Index, Layout, KIND_U32, KIND_U64, KIND_BYTES, LIB_PATH,
    cuart_build, cuart_destroy, cuart_dump, cuart_get_error, cuart_launch_count, cuart_layout_build,
    cuart_layout_free, cuart_layout_lookup, cuart_layout_sectors, cuart_layout_view_get, cuart_lookup, cuart_lookup_host,
    cuart_stats, cuart_status_string, cuart_update, cuart_update_host, cuart_upload, lib,
    cuart_update_ex, cuart_erase, cuart_free_leaves, cuart_range,
    PREBUCKET_AUTO, PREBUCKET_OFF, PREBUCKET_ON, SLICE_AUTO, SLICE_OFF, SLICE_ON, WIDE_AUTO, WIDE_OFF, WIDE_ON,
    BUCKET_FORM_AUTO, BUCKET_GLOBAL, BUCKET_TILE,
    cuart_kernel_timer, cuart_kernel_time, cuart_kernel_time_ex, LongIndex, pack_long,
)
