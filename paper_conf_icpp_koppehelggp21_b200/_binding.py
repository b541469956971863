"""ctypes marshalling for libcuart.so (see include/cuart.h for the contract)."""
from __future__ import annotations

import ctypes
import os

import numpy as np

LIB_PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), "libcuart.so")
CUART_MISS = 0xFFFFFFFFFFFFFFFF
CUART_MAX_KEY = 32
KIND_U32, KIND_U64, KIND_BYTES = 1, 2, 3
CUART_LUT_AUTO = 0xFFFFFFFF
LUT_FORMAT_AUTO, LUT_LINKS, LUT_COMPACT32, LUT_RANK = 0, 1, 2, 3


class CuartError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        super().__init__(f"{where}: cuart status {status} ({cuart_status_string(status)})")


class _Keys(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int), ("data", ctypes.c_void_p), ("lengths", ctypes.c_void_p)]


class _Opts(ctypes.Structure):
    _fields_ = [("lut_bytes", ctypes.c_uint32), ("l2_persist", ctypes.c_uint32),
                ("device", ctypes.c_int32), ("lut_format", ctypes.c_uint32), ("prebucket", ctypes.c_uint32), ("slice_lut", ctypes.c_uint32), ("wide_lut", ctypes.c_uint32),
                ("bucket_form", ctypes.c_uint32), ("skip_log2", ctypes.c_uint32)]


class _Stats(ctypes.Structure):
    _fields_ = [("count", ctypes.c_uint64 * 8), ("bytes", ctypes.c_uint64 * 8), ("n_keys", ctypes.c_uint64),
                ("lut_entries", ctypes.c_uint64), ("lut_bytes_total", ctypes.c_uint64),
                ("arena_bytes", ctypes.c_uint64), ("lut_bytes", ctypes.c_uint32), ("key_kind", ctypes.c_uint32),
                ("root", ctypes.c_uint64), ("max_depth", ctypes.c_uint32), ("lut_format", ctypes.c_uint32),
                ("lut_exceptions", ctypes.c_uint64), ("wide_lut", ctypes.c_uint32), ("l2_window_bytes", ctypes.c_uint64),
                ("skip_prefix", ctypes.c_uint32), ("skip_slots", ctypes.c_uint64)]


class _View(ctypes.Structure):
    _fields_ = [("buf", ctypes.c_void_p * 8), ("count", ctypes.c_uint64 * 8), ("record_bytes", ctypes.c_uint64 * 8),
                ("lut", ctypes.c_void_p), ("lut_entries", ctypes.c_uint64), ("root", ctypes.c_uint64),
                ("lut_bytes", ctypes.c_uint32), ("key_kind", ctypes.c_uint32), ("n_keys", ctypes.c_uint64)]


_lib = None


def lib():
    """Load libcuart.so; raises if it was not built (no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run `python -m paper_conf_icpp_koppehelggp21_b200.build`")
        L = ctypes.CDLL(LIB_PATH)
        P, S, I = ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int
        sig = {
            "cuart_build": [P, P, S, P, P], "cuart_lookup": [P, P, S, P, P], "cuart_update": [P, P, P, S, P],
            "cuart_destroy": [P], "cuart_update_ex": [P, P, P, P, S, P], "cuart_erase": [P, P, S, P],
            "cuart_free_leaves": [P, P, S, P], "cuart_range": [P, P, P, S, P, P],
            "cuart_kernel_timer": [P, I], "cuart_kernel_time": [P, P, P, P], "cuart_kernel_time_ex": [P, P, P, P, P], "cuart_lookup_host": [P, P, S, P], "cuart_update_host": [P, P, P, S],
            "cuart_stats": [P, P], "cuart_dump": [P, P], "cuart_get_error": [P],
            "cuart_layout_build": [P, P, S, P, P], "cuart_layout_view_get": [P, P],
            "cuart_layout_lookup": [P, P, S, P, I], "cuart_layout_sectors": [P, P, S, P, I], "cuart_layout_sectors_ex": [P, P, S, P, I, ctypes.c_uint32], "cuart_upload": [P, P, P], "cuart_layout_free": [P],
        }
        for name, args in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = ctypes.c_int
        L.cuart_status_string.argtypes = [ctypes.c_int]
        L.cuart_status_string.restype = ctypes.c_char_p
        L.cuart_route_scratch_bytes.argtypes = [S, ctypes.c_uint32]
        L.cuart_route_scratch_bytes.restype = S
        L.cuart_route.argtypes = [P, S, P, ctypes.c_uint32, P, P, P, P, P, P, P, P]
        L.cuart_route.restype = ctypes.c_int
        L.cuart_partition_by_flag.argtypes = [P, S, P, P, P, P, P, P, P, P, P]
        L.cuart_partition_by_flag.restype = ctypes.c_int
        L.cuart_unroute.argtypes = [P, P, S, P, P]
        L.cuart_unroute.restype = ctypes.c_int
        U32 = ctypes.c_uint32
        for name, args in {"cuart_build_long": [P, P, P, S, P, P], "cuart_lookup_long": [P, P, P, S, P, P],
                           "cuart_update_long": [P, P, P, P, S, P]}.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = ctypes.c_int
        L.cuart_debug_set_epoch.argtypes = [P, ctypes.c_uint32]
        L.cuart_debug_set_epoch.restype = ctypes.c_int
        L.cuart_fill_miss.argtypes = [P, S, P]
        L.cuart_fill_miss.restype = ctypes.c_int
        L.cuart_launch_count.argtypes = []
        L.cuart_launch_count.restype = ctypes.c_uint64
        _lib = L
    return _lib


def cuart_status_string(s: int) -> str:
    return lib().cuart_status_string(int(s)).decode()


def cuart_launch_count() -> int:
    return int(lib().cuart_launch_count())


def _check(rc, where):
    if rc != 0:
        raise CuartError(rc, where)


# ------------------------------------------------------------------ marshalling
def _is_torch(x):
    return type(x).__module__.startswith("torch")


def _ptr(x):
    if x is None:
        return None
    if _is_torch(x):
        return x.data_ptr()
    return x.ctypes.data


def _kind_of(x):
    dt = str(x.dtype)
    if dt.endswith(("uint64", "int64")):
        return KIND_U64
    if dt.endswith(("uint32", "int32")):
        return KIND_U32
    if dt.endswith("uint8") and len(x.shape) == 2:
        return KIND_BYTES
    raise TypeError(f"unsupported key array dtype/shape {x.dtype} {tuple(x.shape)}")


def _contig(x):
    if _is_torch(x):
        return x.contiguous()
    return np.ascontiguousarray(x)


def _check_dev(t, device=None, what="tensor"):
    """A device-pointer argument: a contiguous CUDA tensor (on `device` if given)."""
    if not _is_torch(t) or not t.is_cuda:
        raise ValueError(f"{what} must be a CUDA tensor (device pointer)")
    if not t.is_contiguous():
        raise ValueError(f"{what} must be contiguous")
    if device is not None and t.device != device:
        raise ValueError(f"{what} is on {t.device}, the index on {device}")


def _check_out(out, n, device=None, width=8):
    """The result buffer the kernels write n x `width` bytes into, in a row."""
    _check_dev(out, device, "out")
    if out.element_size() != width or out.dim() < 1:
        raise ValueError(f"out must have {width}-byte elements")
    if out.numel() < n * (out.shape[-1] if out.dim() == 2 else 1) or out.shape[0] < n:
        raise ValueError("out too small")


def make_keys(keys, lengths=None):
    """keys: u64/u32 array, or (slots uint8[n,32], lengths uint8[n]) / slots + lengths."""
    if isinstance(keys, tuple):
        keys, lengths = keys
    keys = _contig(keys)
    kind = _kind_of(keys)
    if kind == KIND_BYTES:
        if lengths is None:
            raise ValueError("byte-string keys need lengths")
        if keys.shape[1] != CUART_MAX_KEY:
            raise ValueError("byte-string keys must be 32-byte slots")
        lengths = _contig(lengths)
    n = int(keys.shape[0])
    st = _Keys(kind, _ptr(keys), _ptr(lengths) if kind == KIND_BYTES else None)
    return st, n, (keys, lengths)


PREBUCKET_AUTO, PREBUCKET_OFF, PREBUCKET_ON = 0, 1, 2
SLICE_AUTO, SLICE_OFF, SLICE_ON = 0, 1, 2
WIDE_AUTO, WIDE_OFF, WIDE_ON = 0, 1, 2
BUCKET_FORM_AUTO, BUCKET_GLOBAL, BUCKET_TILE = 0, 1, 2


def _opts(lut_bytes=CUART_LUT_AUTO, l2_persist=0, device=-1, lut_format=0, prebucket=0, slice_lut=0, wide_lut=0,
          bucket_form=0, skip_log2=0):
    return _Opts(lut_bytes, l2_persist, device, lut_format, prebucket, slice_lut, wide_lut, bucket_form, skip_log2)


def _stream_ptr(stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


# ------------------------------------------------------------------ hot path
def cuart_build(keys, values, lut_bytes=CUART_LUT_AUTO, l2_persist=0, device=-1, lut_format=0, prebucket=0,
                slice_lut=0, wide_lut=0, bucket_form=0, skip_log2=0):
    """Build + upload (host buffers).  Returns an opaque handle (int)."""
    k, n, keep = make_keys(keys)
    v = np.ascontiguousarray(values, dtype=np.uint64)
    if v.shape[0] != n:
        raise ValueError("values length mismatch")
    h = ctypes.c_void_p()
    o = _opts(lut_bytes, l2_persist, device, lut_format, prebucket, slice_lut, wide_lut, bucket_form, skip_log2)
    _check(lib().cuart_build(ctypes.byref(k), _ptr(v), n, ctypes.byref(o), ctypes.byref(h)), "cuart_build")
    return h.value


def _dev_keys(keys, device=None):
    """make_keys for a device batch: the key (and length) tensors are checked to be
    contiguous CUDA tensors on the index's device."""
    k, n, keep = make_keys(keys)
    _check_dev(keep[0], device, "keys")
    if keep[1] is not None:
        _check_dev(keep[1], device, "lengths")
    return k, n, keep


def cuart_lookup(h, queries, out, stream=None, device=None):
    """Device buffers (torch CUDA tensors); async on `stream` (default: current)."""
    q, n, keep = _dev_keys(queries, device)
    _check_out(out, n, device)
    _check(lib().cuart_lookup(h, ctypes.byref(q), n, _ptr(out), _stream_ptr(stream)), "cuart_lookup")
    return out


def cuart_update(h, keys, new_values, stream=None, device=None):
    k, n, keep = _dev_keys(keys, device)
    _check_dev(new_values, device, "new_values")
    if new_values.shape[0] != n or new_values.element_size() != 8:
        raise ValueError("new_values must be n 8-byte values")
    _check(lib().cuart_update(h, ctypes.byref(k), _ptr(new_values), n, _stream_ptr(stream)), "cuart_update")


def cuart_update_ex(h, keys, new_values, is_delete, stream=None, device=None):
    """Mixed batch: is_delete (device uint8[n]) marks deletes (reading C17)."""
    k, n, keep = _dev_keys(keys, device)
    _check_dev(new_values, device, "new_values")
    _check_dev(is_delete, device, "is_delete")
    if new_values.shape[0] != n or new_values.element_size() != 8 or is_delete.shape[0] != n or \
            is_delete.element_size() != 1:
        raise ValueError("new_values / is_delete must be n 8-byte / 1-byte elements")
    _check(lib().cuart_update_ex(h, ctypes.byref(k), _ptr(new_values), _ptr(is_delete), n,
                                 _stream_ptr(stream)), "cuart_update_ex")


def cuart_erase(h, keys, stream=None, device=None):
    k, n, keep = _dev_keys(keys, device)
    _check(lib().cuart_erase(h, ctypes.byref(k), n, _stream_ptr(stream)), "cuart_erase")


def cuart_range(h, lo, hi, bounds, stream=None, device=None):
    """bounds: device uint64/int64 tensor [n, 6] (start/end per leaf class)."""
    kl, n, keep1 = _dev_keys(lo, device)
    kh, n2, keep2 = _dev_keys(hi, device)
    if n2 != n:
        raise ValueError("lo/hi length mismatch")
    _check_dev(bounds, device, "bounds")
    if bounds.element_size() != 8 or bounds.numel() < 6 * n:
        raise ValueError("bounds must hold 6 x n 8-byte entries")
    _check(lib().cuart_range(h, ctypes.byref(kl), ctypes.byref(kh), n, _ptr(bounds), _stream_ptr(stream)), "cuart_range")
    return bounds


def cuart_kernel_timer(h, enable=True):
    _check(lib().cuart_kernel_timer(h, 1 if enable else 0), "cuart_kernel_timer")


def cuart_kernel_time(h):
    """(total_ms, launches, lookups) of k_lookup since the timer was enabled; resets."""
    t, l, q = ctypes.c_double(), ctypes.c_uint64(), ctypes.c_uint64()
    _check(lib().cuart_kernel_time(h, ctypes.byref(t), ctypes.byref(l), ctypes.byref(q)), "cuart_kernel_time")
    return t.value, l.value, q.value


def cuart_kernel_time_ex(h):
    """(total_ms, launches, lookups, slice_launches): as cuart_kernel_time, plus how many
    timed launches were k_lookup_slice (the bucketed walk with the smem table slice)."""
    t, l, q, sl = ctypes.c_double(), ctypes.c_uint64(), ctypes.c_uint64(), ctypes.c_uint64()
    _check(lib().cuart_kernel_time_ex(h, ctypes.byref(t), ctypes.byref(l), ctypes.byref(q), ctypes.byref(sl)),
           "cuart_kernel_time_ex")
    return t.value, l.value, q.value, sl.value


def cuart_free_leaves(h):
    cnt = ctypes.c_size_t()
    _check(lib().cuart_free_leaves(h, None, 0, ctypes.byref(cnt)), "cuart_free_leaves")
    ids = np.zeros(max(1, cnt.value), dtype=np.uint32)
    _check(lib().cuart_free_leaves(h, _ptr(ids), cnt.value, ctypes.byref(cnt)), "cuart_free_leaves")
    return ids[: cnt.value]


def cuart_lookup_host(h, queries, out=None):
    q, n, keep = make_keys(queries)
    if out is None:
        out = np.empty(n, dtype=np.uint64)
    _check(lib().cuart_lookup_host(h, ctypes.byref(q), n, _ptr(out)), "cuart_lookup_host")
    return out


def cuart_update_host(h, keys, new_values):
    k, n, keep = make_keys(keys)
    v = _contig(new_values)
    _check(lib().cuart_update_host(h, ctypes.byref(k), _ptr(v), n), "cuart_update_host")


def cuart_destroy(h):
    if h:
        _check(lib().cuart_destroy(h), "cuart_destroy")


def cuart_get_error(h) -> int:
    return int(lib().cuart_get_error(h))


def cuart_stats(h) -> dict:
    s = _Stats()
    _check(lib().cuart_stats(h, ctypes.byref(s)), "cuart_stats")
    return _stats_dict(s)


def _stats_dict(s):
    names = {1: "n4", 2: "n16", 3: "n48", 4: "n256", 5: "leaf8", 6: "leaf16", 7: "leaf32"}
    d = {names[t]: int(s.count[t]) for t in names}
    d.update({f"{names[t]}_bytes": int(s.bytes[t]) for t in names})
    d.update(n_keys=int(s.n_keys), lut_bytes=int(s.lut_bytes), lut_entries=int(s.lut_entries),
             arena_bytes=int(s.arena_bytes), root=int(s.root), max_depth=int(s.max_depth), key_kind=int(s.key_kind),
             lut_format=int(s.lut_format), lut_exceptions=int(s.lut_exceptions), wide_lut=int(s.wide_lut),
             l2_window_bytes=int(s.l2_window_bytes), skip_prefix=int(s.skip_prefix), skip_slots=int(s.skip_slots))
    return d


# ------------------------------------------------------------------ host layout
def cuart_layout_build(keys, values, lut_bytes=0):
    k, n, keep = make_keys(keys)
    v = np.ascontiguousarray(values, dtype=np.uint64)
    if v.shape[0] != n:
        raise ValueError("values length mismatch")
    h = ctypes.c_void_p()
    o = _opts(lut_bytes)
    _check(lib().cuart_layout_build(ctypes.byref(k), _ptr(v), n, ctypes.byref(o), ctypes.byref(h)), "cuart_layout_build")
    return h.value


def cuart_layout_free(l):
    if l:
        lib().cuart_layout_free(l)


def cuart_layout_view_get(l) -> dict:
    """Copies of the layout's arrays as numpy (record bytes per type code, LUT, root)."""
    v = _View()
    _check(lib().cuart_layout_view_get(l, ctypes.byref(v)), "cuart_layout_view_get")
    bufs = {}
    for t in range(1, 8):
        nbytes = int(v.count[t]) * int(v.record_bytes[t])
        if nbytes:
            bufs[t] = np.ctypeslib.as_array((ctypes.c_uint8 * nbytes).from_address(v.buf[t])).copy()
        else:
            bufs[t] = np.zeros(0, np.uint8)
    lut = None
    if v.lut:
        lut = np.ctypeslib.as_array((ctypes.c_uint64 * int(v.lut_entries)).from_address(v.lut)).copy()
    return {"buf": bufs, "count": [int(v.count[t]) for t in range(8)],
            "record_bytes": [int(v.record_bytes[t]) for t in range(8)], "lut": lut, "root": int(v.root),
            "lut_bytes": int(v.lut_bytes), "key_kind": int(v.key_kind), "n_keys": int(v.n_keys)}


def cuart_layout_lookup(l, queries, threads=0):
    q, n, keep = make_keys(queries)
    out = np.empty(n, dtype=np.uint64)
    _check(lib().cuart_layout_lookup(l, ctypes.byref(q), n, _ptr(out), threads), "cuart_layout_lookup")
    return out


def cuart_layout_sectors(l, queries, threads=0, wide=False, skip_prefix=0):
    q, n, keep = make_keys(queries)
    out = np.empty(n, dtype=np.uint32)
    flags = (1 if wide else 0) | ((int(skip_prefix) & 0xFF) << 8)
    _check(lib().cuart_layout_sectors_ex(l, ctypes.byref(q), n, _ptr(out), threads, flags),
           "cuart_layout_sectors_ex")
    return out


def cuart_upload(l, lut_bytes=0, l2_persist=0, device=-1, lut_format=0, prebucket=0, slice_lut=0, wide_lut=0,
                 bucket_form=0, skip_log2=0):
    h = ctypes.c_void_p()
    o = _opts(lut_bytes, l2_persist, device, lut_format, prebucket, slice_lut, wide_lut, bucket_form, skip_log2)
    _check(lib().cuart_upload(l, ctypes.byref(o), ctypes.byref(h)), "cuart_upload")
    return h.value


def cuart_dump(h):
    """Device -> host snapshot of every array; returns a layout handle (free with cuart_layout_free)."""
    l = ctypes.c_void_p()
    _check(lib().cuart_dump(h, ctypes.byref(l)), "cuart_dump")
    return l.value


# ------------------------------------------------------------------ object wrappers
class Layout:
    """Host-resident flattened layout (no GPU needed)."""

    def __init__(self, keys, values, lut_bytes=0):
        self.h = cuart_layout_build(keys, values, lut_bytes)

    def lookup(self, queries, threads=0):
        return cuart_layout_lookup(self.h, queries, threads)

    def view(self):
        return cuart_layout_view_get(self.h)

    def sectors(self, queries, threads=0, wide=False, skip_prefix=0):
        return cuart_layout_sectors(self.h, queries, threads, wide, skip_prefix)

    def close(self):
        cuart_layout_free(self.h)
        self.h = None

    def __del__(self):
        try:
            if self.h:
                self.close()
        except Exception:
            pass


def _torch_device(device):
    """The CUDA device the library put the index on (-1 = the current device)."""
    try:
        import torch
        if not torch.cuda.is_available():
            return None
        return torch.device("cuda", torch.cuda.current_device() if device is None or device < 0 else device)
    except Exception:        # noqa: BLE001 -- no torch / no CUDA: the C library reports NO_DEVICE itself
        return None


class Index:
    """Device-resident CuART index on one GPU."""

    def __init__(self, keys, values, lut_bytes=CUART_LUT_AUTO, l2_persist=0, device=-1, lut_format=0, prebucket=0,
                 slice_lut=0, wide_lut=0, bucket_form=0, skip_log2=0):
        self.h = cuart_build(keys, values, lut_bytes, l2_persist, device, lut_format, prebucket, slice_lut, wide_lut,
                             bucket_form, skip_log2)
        self.device = _torch_device(device)

    @classmethod
    def from_layout(cls, layout: "Layout", l2_persist=0, device=-1, lut_format=0, prebucket=0, slice_lut=0,
                    wide_lut=0, bucket_form=0, skip_log2=0):
        """Upload an already-built host layout (keeps the host copy usable)."""
        self = cls.__new__(cls)
        self.h = cuart_upload(layout.h, 0, l2_persist, device, lut_format, prebucket, slice_lut, wide_lut, bucket_form,
                              skip_log2)
        self.device = _torch_device(device)
        return self

    def lookup(self, queries, out=None, stream=None):
        import torch
        if out is None:
            q = queries[0] if isinstance(queries, tuple) else queries
            out = torch.empty(q.shape[0], dtype=torch.uint64, device=q.device)
        return cuart_lookup(self.h, queries, out, stream, getattr(self, "device", None))

    def update(self, keys, new_values, stream=None):
        cuart_update(self.h, keys, new_values, stream, getattr(self, "device", None))

    def update_ex(self, keys, new_values, is_delete, stream=None):
        cuart_update_ex(self.h, keys, new_values, is_delete, stream, getattr(self, "device", None))

    def erase(self, keys, stream=None):
        cuart_erase(self.h, keys, stream, getattr(self, "device", None))

    def free_leaves(self):
        return cuart_free_leaves(self.h)

    def range(self, lo, hi, bounds=None, stream=None):
        import torch
        if bounds is None:
            l0 = lo[0] if isinstance(lo, tuple) else lo
            bounds = torch.empty((l0.shape[0], 6), dtype=torch.int64, device=l0.device)
        return cuart_range(self.h, lo, hi, bounds, stream, getattr(self, "device", None))

    def lookup_host(self, queries, out=None):
        return cuart_lookup_host(self.h, queries, out)

    def update_host(self, keys, new_values):
        cuart_update_host(self.h, keys, new_values)

    def stats(self):
        return cuart_stats(self.h)

    def dump(self):
        l = cuart_dump(self.h)
        try:
            return cuart_layout_view_get(l)
        finally:
            cuart_layout_free(l)

    def dump_layout(self):
        return cuart_dump(self.h)

    def get_error(self):
        return cuart_get_error(self.h)

    def close(self):
        if self.h:
            cuart_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


# ------------------------------------------------------------------ f4: keys longer than 32 bytes
def pack_long(keys):
    """list of bytes -> (data uint8[total], offsets uint64[n+1]) (packed form of the *_long calls)."""
    lens = np.fromiter((len(k) for k in keys), dtype=np.uint64, count=len(keys))
    offsets = np.zeros(len(keys) + 1, dtype=np.uint64)
    np.cumsum(lens, out=offsets[1:])
    data = np.frombuffer(b"".join(keys), dtype=np.uint8) if keys else np.zeros(1, np.uint8)
    return np.ascontiguousarray(data), offsets


class LongIndex:
    """CUART_KEY_LONG index (§8(f) f4, P:126 option 2): keys of 1..255 bytes; leaves of
    keys > 32 bytes live in host memory and the host finishes their compares."""

    def __init__(self, keys, values, lut_bytes=0, device=-1):
        data, off = pack_long(keys)
        v = np.ascontiguousarray(values, dtype=np.uint64)
        if v.shape[0] != len(keys):
            raise ValueError("values length mismatch")
        h = ctypes.c_void_p()
        o = _opts(lut_bytes, 0, device, 0, 0, 0, 0)
        _check(lib().cuart_build_long(_ptr(data), _ptr(off), _ptr(v), len(keys), ctypes.byref(o), ctypes.byref(h)),
               "cuart_build_long")
        self.h = h.value

    def lookup(self, queries):
        data, off = pack_long(queries)
        out = np.empty(len(queries), dtype=np.uint64)
        _check(lib().cuart_lookup_long(self.h, _ptr(data), _ptr(off), len(queries), _ptr(out), None),
               "cuart_lookup_long")
        return out

    def update(self, keys, values):
        data, off = pack_long(keys)
        v = np.ascontiguousarray(values, dtype=np.uint64)
        _check(lib().cuart_update_long(self.h, _ptr(data), _ptr(off), _ptr(v), len(keys), None), "cuart_update_long")

    def close(self):
        if self.h:
            cuart_destroy(self.h)
            self.h = None
