"""Multi-GPU layer: argument marshalling for the cuart_dist_* C ABI.

The protocol -- range partitioning by the first 8 key bytes, K-ROUTE fused with
K-BUCKET on the source, the count exchange, the fused push into the owners'
receive windows over NVLink (transport ``p2p``) or the grouped ncclSend/ncclRecv
baseline (transport ``nccl``), the owner's walk, the fused return and the gather,
chunk pipelining with device-side arrival flags, replica mode -- lives in
``csrc/dist.cu`` (see include/cuart.h for the contract).  This module only

* builds the ``cuart_dist_cfg`` (rank / world size of a torch.distributed group,
  the NCCL unique id broadcast from rank 0),
* supplies the host bootstrap collective the library calls during build and
  teardown (an all-gather of a few hundred bytes: window handles, splitters)
  through ``torch.distributed`` (NCCL on the GPU box; gloo in the tests), or
  through a thread barrier for virtual ranks in one process,
* passes tensor pointers and the current stream.

Config 5's mixed rounds (reading C7) are three C-ABI calls: cuart_partition_by_flag
splits a round into lookups and updates, cuart_dist_lookup / cuart_dist_update run
them, cuart_unroute restores op order.
"""
from __future__ import annotations

import ctypes
import threading

import numpy as np
import torch
import torch.distributed as dist

from . import _binding as B

MODES = {"replica": 1, "range": 2}
TRANSPORTS = {"nccl": 1, "p2p": 2}
MAX_RANKS = 16
AllGatherFn = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t)


class _DistCfg(ctypes.Structure):
    _fields_ = [("rank", ctypes.c_int32), ("nranks", ctypes.c_int32), ("mode", ctypes.c_uint32),
                ("transport", ctypes.c_uint32), ("nccl_id", ctypes.c_uint8 * 128),
                ("allgather", AllGatherFn), ("allgather_ctx", ctypes.c_void_p),
                ("splitters", ctypes.c_void_p), ("keys_local", ctypes.c_uint32), ("reserved0", ctypes.c_uint32),
                ("chunk", ctypes.c_uint64), ("opts", B._Opts)]


def _sig(L):
    P, S, U32 = ctypes.c_void_p, ctypes.c_size_t, ctypes.c_uint32
    for name, args in {"cuart_dist_unique_id": [P], "cuart_dist_build": [P, P, P, S, P],
                       "cuart_dist_lookup": [P, P, S, P, P], "cuart_dist_update": [P, P, P, S, P],
                       "cuart_dist_partition": [P, P, S, P, P], "cuart_dist_chunk_plan": [U32, U32, P, P, P, P],
                       "cuart_dist_last": [P, P, P], "cuart_dist_mixed": [P, P, P, P, S, P, P]}.items():
        f = getattr(L, name)
        if f.argtypes is None:
            f.argtypes = args
            f.restype = ctypes.c_int
    return L


def lib():
    return _sig(B.lib())


# ------------------------------------------------------------------ bootstrap collectives
class TorchAllGather:
    """Host all-gather over a torch.distributed group (bytes in, rank-ordered bytes out)."""

    def __init__(self, group=None):
        self.group = group

    def __call__(self, payload: bytes) -> list[bytes]:
        out = [None] * dist.get_world_size(self.group)
        dist.all_gather_object(out, payload, group=self.group)
        return out


class ThreadAllGather:
    """All-gather between `world` threads of one process (virtual ranks sharing a GPU)."""

    def __init__(self, world):
        self.world = world
        self.slots = [None] * world
        self.barrier = threading.Barrier(world)

    def bind(self, rank):
        def gather(payload: bytes) -> list[bytes]:
            self.slots[rank] = payload
            self.barrier.wait()
            out = list(self.slots)
            self.barrier.wait()
            return out
        return gather


def _callback(gather):
    def cb(ctx, send, recv, nbytes):
        try:
            parts = gather(ctypes.string_at(send, nbytes))
            buf = b"".join(parts)
            if len(buf) != nbytes * len(parts):
                return 1
            ctypes.memmove(recv, buf, len(buf))
            return 0
        except Exception:          # noqa: BLE001 -- a failed collective is reported as CUART_ERR_NCCL
            return 1
    return AllGatherFn(cb)


def unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    B._check(lib().cuart_dist_unique_id(buf), "cuart_dist_unique_id")
    return buf.raw


def _cfg(rank, world, mode, transport, gather, nccl_id=None, splitters=None, keys_local=False, chunk=0, opts=None):
    c = _DistCfg()
    c.rank, c.nranks = rank, world
    c.mode, c.transport = MODES[mode], TRANSPORTS[transport]
    if nccl_id is not None:
        ctypes.memmove(c.nccl_id, nccl_id, 128)
    keep = []
    if gather is not None:
        fn = _callback(gather)
        keep.append(fn)
        c.allgather = fn
    if splitters is not None and world > 1:
        sp = np.ascontiguousarray(splitters, dtype=np.uint64)
        keep.append(sp)
        c.splitters = sp.ctypes.data
    c.keys_local = 1 if keys_local else 0
    c.chunk = int(chunk)
    c.opts = opts if opts is not None else B._opts(3)
    return c, keep


def partition(keys, rank, world, mode="range", splitters=None, gather=None):
    """cuart_dist_partition: (splitters uint64[world-1], owner uint8[n]) on the host."""
    k, n, keep = B.make_keys(keys)
    c, keep2 = _cfg(rank, world, mode, "p2p", gather, splitters=splitters)
    sp = np.zeros(max(1, world - 1), np.uint64)
    own = np.zeros(max(1, n), np.uint8)
    B._check(lib().cuart_dist_partition(ctypes.byref(c), ctypes.byref(k), n, sp.ctypes.data, own.ctypes.data),
             "cuart_dist_partition")
    return sp[: world - 1], own[:n]


def chunk_plan(M, me):
    """cuart_dist_chunk_plan: (seg_start[P+1], res_off[P], push_off[P]) for rank `me`."""
    M = np.ascontiguousarray(M, dtype=np.uint64)
    P = M.shape[0]
    seg, res, push = np.zeros(P + 1, np.uint64), np.zeros(P, np.uint64), np.zeros(P, np.uint64)
    B._check(lib().cuart_dist_chunk_plan(P, me, M.ctypes.data, seg.ctypes.data, res.ctypes.data, push.ctypes.data),
             "cuart_dist_chunk_plan")
    return seg, res, push


# ------------------------------------------------------------------ host helpers (bench / tests)
def prefix8(keys) -> np.ndarray:
    """First 8 key bytes read big-endian, as uint64 (numeric order = key order)."""
    if isinstance(keys, tuple):
        slots, lens = keys
        head = np.asarray(slots, np.uint8)[:, :8].copy()
        head[np.arange(8)[None, :] >= np.asarray(lens, np.uint8)[:, None]] = 0
        return np.ascontiguousarray(head).view(">u8").ravel().astype(np.uint64)
    keys = np.asarray(keys)
    if keys.dtype == np.uint32:
        return keys.astype(np.uint64) << np.uint64(32)
    return keys.astype(np.uint64)


def owners(prefix: np.ndarray, splitters: np.ndarray) -> np.ndarray:
    return np.searchsorted(splitters, prefix, side="right").astype(np.int64)


def select(keys, mask):
    if isinstance(keys, tuple):
        return (keys[0][mask], keys[1][mask])
    return keys[mask]


# ------------------------------------------------------------------ the distributed index
class DistIndex:
    """A CuART index spread over the ranks of a group (cuart_dist_build)."""

    def __init__(self, keys, values, mode="range", transport="p2p", group=None, splitters=None, keys_local=False,
                 chunk=0, lut_bytes=3, device=None, rank=None, world=None, gather=None, nccl_id=None, **opts):
        """keys/values: host arrays -- the GLOBAL key set (identical on every rank), or
        with keys_local=True this rank's share of the partition `splitters`.
        rank/world/gather default to the torch.distributed group."""
        if rank is None:
            rank, world = dist.get_rank(group), dist.get_world_size(group)
        if gather is None and world > 1:
            gather = TorchAllGather(group)
        if nccl_id is None and world > 1 and transport == "nccl":
            obj = [unique_id() if rank == 0 else None]
            dist.broadcast_object_list(obj, src=0, group=group)
            nccl_id = obj[0]
        dev = torch.cuda.current_device() if device is None else torch.device(device).index or 0
        self.device = torch.device("cuda", dev)
        self.mode, self.transport, self.rank, self.world = mode, transport, rank, world
        k, n, keepk = B.make_keys(keys)
        v = np.ascontiguousarray(values, dtype=np.uint64)
        if v.shape[0] != n:
            raise ValueError("values length mismatch")
        c, self._keep = _cfg(rank, world, mode, transport, gather, nccl_id, splitters, keys_local, chunk,
                             B._opts(lut_bytes, device=dev, **opts))
        if mode == "range" and world > 1:
            self.splitters = (np.ascontiguousarray(splitters, np.uint64) if splitters is not None
                              else partition(keys, rank, world)[0])
        else:
            self.splitters = np.zeros(0, np.uint64)
        h = ctypes.c_void_p()
        B._check(lib().cuart_dist_build(ctypes.byref(c), ctypes.byref(k), v.ctypes.data, n, ctypes.byref(h)),
                 "cuart_dist_build")
        self.h = h.value
        self.index = B.Index.__new__(B.Index)       # the local part (stats, dump, timers)
        self.index.h = self.h

    def lookup(self, queries, out=None, stream=None):
        q, n, keep = B.make_keys(queries)
        if out is None:
            out = torch.empty(n, dtype=torch.int64, device=self.device)
        B._check_out(out, n, self.device)
        B._check(lib().cuart_dist_lookup(self.h, ctypes.byref(q), n, out.data_ptr(), B._stream_ptr(stream)),
                 "cuart_dist_lookup")
        return out

    def update(self, keys, values, stream=None):
        k, n, keep = B.make_keys(keys)
        values = values.contiguous()
        if values.shape[0] != n:
            raise ValueError("values length mismatch")
        B._check_dev(values, self.device, "values")
        B._check(lib().cuart_dist_update(self.h, ctypes.byref(k), values.data_ptr(), n, B._stream_ptr(stream)),
                 "cuart_dist_update")

    def mixed_round(self, keys, values, is_update, lens=None, stream=None, events=None, fused=False):
        """One round of a mixed op stream (reading C7): every lookup sees the state
        before the round; the round's updates then apply in global (rank-major, op)
        order.  Returns per op the lookup result, CUART_MISS for update ops.
        Default: cuart_partition_by_flag, cuart_dist_lookup, cuart_dist_update,
        cuart_unroute (events: optional 5 CUDA events recorded around those four
        calls -- measurement only).  fused=True (range mode): one cuart_dist_mixed
        call whose two passes filter their op kind -- measured slower on c5
        (DESIGN.md §10), kept as an API."""
        if fused and self.mode == "range":
            kk, n, keep = B.make_keys((keys, lens) if lens is not None else keys)
            out = torch.empty(n, dtype=torch.int64, device=keys.device)
            B._check_dev(values, self.device, "values")
            B._check_dev(is_update, self.device, "is_update")
            if events:
                events[0].record()
            B._check(lib().cuart_dist_mixed(self.h, ctypes.byref(kk), values.data_ptr(), is_update.data_ptr(), n,
                                            out.data_ptr(), B._stream_ptr(stream)), "cuart_dist_mixed")
            if events:
                events[-1].record()
            return out
        rec = (lambda i: events[i].record()) if events else (lambda i: None)
        rec(0)
        n = keys.shape[0]
        ok, ol, ov = torch.empty_like(keys), (torch.empty_like(lens) if lens is not None else None), torch.empty_like(values)
        perm = torch.empty(n, dtype=torch.int32, device=keys.device)
        counts = torch.empty(2, dtype=torch.int64, device=keys.device)
        scratch = torch.empty(max(1, B.lib().cuart_route_scratch_bytes(n, 2)), dtype=torch.uint8, device=keys.device)
        kk, _, keep = B.make_keys((keys, lens) if lens is not None else keys)
        sp = B._stream_ptr(stream)
        B._check(B.lib().cuart_partition_by_flag(ctypes.byref(kk), n, is_update.data_ptr(), values.data_ptr(),
                                                 ok.data_ptr(), ol.data_ptr() if ol is not None else None,
                                                 ov.data_ptr(), perm.data_ptr(), counts.data_ptr(), scratch.data_ptr(),
                                                 sp), "cuart_partition_by_flag")
        rec(1)
        n_l = int(counts[0].item())                  # host needs the split to size the two calls
        res = torch.empty(n, dtype=torch.int64, device=keys.device)
        B._check(B.lib().cuart_fill_miss(res.data_ptr() + 8 * n_l, n - n_l, sp), "cuart_fill_miss")
        self.lookup((ok[:n_l], ol[:n_l]) if ol is not None else ok[:n_l], res[:n_l], stream)
        rec(2)
        self.update((ok[n_l:], ol[n_l:]) if ol is not None else ok[n_l:], ov[n_l:], stream)
        rec(3)
        out = torch.empty_like(res)
        B._check(B.lib().cuart_unroute(res.data_ptr(), perm.data_ptr(), n, out.data_ptr(), sp), "cuart_unroute")
        rec(4)
        return out

    def last(self):
        """(ops received as owner, chunks) of this rank's last dist call."""
        r, c = ctypes.c_uint64(), ctypes.c_uint64()
        B._check(lib().cuart_dist_last(self.h, ctypes.byref(r), ctypes.byref(c)), "cuart_dist_last")
        return r.value, c.value

    def stats(self):
        return B.cuart_stats(self.h)

    def close(self):
        """Collective: every rank closes together."""
        if self.h:
            B.cuart_destroy(self.h)              # synchronises this rank's device work first
            self.h = None
            self.index.h = None
