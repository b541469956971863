"""Multi-GPU layer: one process per GPU, torch.distributed for the
plumbing (NCCL over NVLink/NVSwitch on the GPU box), CuART kernels for all data
movement on the device.

Two modes:

* ``replica`` — every rank holds the full index.  Lookups need no exchange: a
  rank serves its own share of the query stream.  Update batches are
  all-gathered and applied everywhere in global (rank-major) order, so replicas
  stay bit-identical.
* ``range``  — the key space is range-partitioned over the first 8 key bytes
  (big-endian) with quantile splitters computed from the key distribution, so
  skewed and dense key sets balance.  Each rank indexes only its range.  A
  batch is routed to the owners (cuart_route: stable per-owner runs + a
  permutation), exchanged with all-to-all (counts, then the runs), served by the
  owner's local index, sent back with the reverse all-to-all and restored to
  query order (cuart_unroute).  Updates travel with their values; because the
  runs of all sources arrive concatenated by source rank and are stable in op
  order, the owner applies them in global rank-major order — the highest global
  op index wins (reading C7).

The protocol is written once against an ``ops`` object: ``CudaOps`` (product,
C-ABI kernels, CUDA tensors, NCCL) or an injected test double (CPU tensors and
the gloo backend) so the exchange logic runs in the CPU test suite.

Range mode has two transports:

* ``nccl`` — route into a local send buffer, then all-to-all of the runs and of
  the results (the library-collective baseline);
* ``p2p``  — fused: every rank maps its peers' receive windows (CUDA IPC over
  NVLink/NVSwitch).  cuart_route_push stores each op straight into its owner's
  window, and the owner's lookup (cuart_lookup_segmented) stores each result
  straight into the requester's result window; only the P x P count matrix goes
  through torch.distributed.  ``p2p_plan`` is the host arithmetic of that
  exchange (pure, CPU-tested).
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist

from . import _binding as B


# ------------------------------------------------------------------ partitioning (host)
def prefix8(keys) -> np.ndarray:
    """First 8 key bytes read big-endian, as uint64 (numeric order = key order)."""
    if isinstance(keys, tuple):
        slots, lens = keys
        slots = np.asarray(slots, np.uint8)
        lens = np.asarray(lens, np.uint8)
        head = slots[:, :8].copy()
        head[np.arange(8)[None, :] >= lens[:, None]] = 0
        return np.ascontiguousarray(head).view(">u8").ravel().astype(np.uint64)
    keys = np.asarray(keys)
    if keys.dtype == np.uint32:
        return keys.astype(np.uint64) << np.uint64(32)
    return keys.astype(np.uint64)


def compute_splitters(sample_prefix: np.ndarray, nparts: int) -> np.ndarray:
    """nparts-1 quantile splitters; owner(k) = number of splitters <= prefix8(k)."""
    if nparts <= 1:
        return np.zeros(0, np.uint64)
    s = np.sort(np.asarray(sample_prefix, np.uint64))
    if s.shape[0] == 0:
        return (np.arange(1, nparts, dtype=np.uint64) * np.uint64((1 << 64) // nparts))
    idx = (np.arange(1, nparts) * s.shape[0]) // nparts
    return s[idx].astype(np.uint64)


def owners(prefix: np.ndarray, splitters: np.ndarray) -> np.ndarray:
    return np.searchsorted(splitters, prefix, side="right").astype(np.int64)


def ks_bytes(kind):
    return {B.KIND_U64: 8, B.KIND_U32: 4, B.KIND_BYTES: 32}[kind]


def select(keys, mask):
    if isinstance(keys, tuple):
        return (keys[0][mask], keys[1][mask])
    return keys[mask]


# ------------------------------------------------------------------ fused p2p exchange: host plan
def p2p_plan(M, rank):
    """Offsets of the fused exchange for `rank`, from the P x P count matrix
    M[s][o] = ops that source s routes to owner o (identical on every rank).

    push_off[o]  : first slot of this rank's run in owner o's receive window
                   (the runs of all sources are concatenated in rank order there);
    seg_start    : [P+1] segments of this rank's receive window by source;
    res_off[s]   : first slot of this rank's results in source s's result window
                   (s keeps its results in owner-major send order);
    need_recv / need_res : window capacities every rank must have (max over ranks).
    """
    M = np.asarray(M, np.int64)
    P = M.shape[0]
    col = M[:, rank]
    return {
        "push_off": [int(M[:rank, o].sum()) for o in range(P)],
        "seg_start": [0] + [int(x) for x in np.cumsum(col)],
        "recv_total": int(col.sum()),
        "res_off": [int(M[s, :rank].sum()) for s in range(P)],
        "need_recv": int(M.sum(axis=0).max()) if P else 0,
        "need_res": int(M.sum(axis=1).max()) if P else 0,
    }


class P2PWindows:
    """This rank's receive windows (keys, lengths, values, results), exported to and
    mapped by every peer (CUDA IPC).  (Re)allocation is collective: every rank calls
    ensure() with the same capacities (derived from the shared count matrix)."""

    def __init__(self, group, world, rank, key_bytes, strings):
        self.group, self.world, self.rank = group, world, rank
        self.kb, self.strings = key_bytes, strings
        self.cap_recv = self.cap_res = 0
        self.own = None          # dict name -> local device address
        self.peer = None         # list over ranks of dict name -> mapped address (own for self)

    def ensure(self, need_recv, need_res):
        if need_recv <= self.cap_recv and need_res <= self.cap_res and self.own is not None:
            return
        self.close()
        self.cap_recv = max(need_recv, 2 * self.cap_recv, 1)
        self.cap_res = max(need_res, 2 * self.cap_res, 1)
        sizes = {"keys": self.cap_recv * self.kb, "vals": self.cap_recv * 8, "res": self.cap_res * 8}
        if self.strings:
            sizes["lens"] = self.cap_recv
        self.own = {k: B.ipc_alloc(v) for k, v in sizes.items()}
        mine = {k: B.ipc_export(v) for k, v in self.own.items()}
        allh = [None] * self.world
        dist.all_gather_object(allh, mine, group=self.group)
        self.peer = [self.own if r == self.rank else {k: B.ipc_import(h) for k, h in allh[r].items()}
                     for r in range(self.world)]

    def close(self):
        if self.peer is not None:
            for r, m in enumerate(self.peer):
                if r != self.rank:
                    for a in m.values():
                        B.ipc_close(a)
        if self.own is not None:
            for a in self.own.values():
                B.ipc_free(a)
        self.own = self.peer = None


# ------------------------------------------------------------------ device ops (product)
class CudaOps:
    """Product ops: CuART C-ABI kernels on CUDA tensors; collectives go over NCCL."""

    def __init__(self, device):
        self.device = torch.device(device)

    def build(self, keys, values, lut_bytes):
        return B.Index(keys, values, lut_bytes=lut_bytes, device=self.device.index or 0)

    def tensor(self, a):
        if isinstance(a, np.ndarray):
            if a.dtype == np.uint64:
                a = a.view(np.int64)
            elif a.dtype == np.uint32:
                a = a.view(np.int32)
            return torch.from_numpy(a).to(self.device)
        return a.to(self.device)

    def route(self, keys, lens, values, splitters, nparts):
        n = keys.shape[0]
        send_keys = torch.empty_like(keys)
        send_lens = torch.empty_like(lens) if lens is not None else None
        send_vals = torch.empty_like(values) if values is not None else None
        perm = torch.empty(n, dtype=torch.int32, device=self.device)
        counts = torch.empty(nparts, dtype=torch.int64, device=self.device)
        scratch = torch.empty(max(1, B.lib().cuart_route_scratch_bytes(n, nparts)), dtype=torch.uint8, device=self.device)
        k, _, keep = B.make_keys((keys, lens) if lens is not None else keys)
        stream = torch.cuda.current_stream(self.device).cuda_stream
        rc = B.lib().cuart_route(B.ctypes.byref(k), n, splitters.data_ptr() if nparts > 1 else None, nparts,
                                 values.data_ptr() if values is not None else None, send_keys.data_ptr(),
                                 send_lens.data_ptr() if send_lens is not None else None,
                                 send_vals.data_ptr() if send_vals is not None else None,
                                 perm.data_ptr(), counts.data_ptr(), scratch.data_ptr(), stream)
        B._check(rc, "cuart_route")
        return send_keys, send_lens, send_vals, perm, counts

    def partition(self, keys, lens, values, flags):
        """Stable split by flag (0 first): cuart_partition_by_flag."""
        n = keys.shape[0]
        ok = torch.empty_like(keys)
        ol = torch.empty_like(lens) if lens is not None else None
        ov = torch.empty_like(values) if values is not None else None
        perm = torch.empty(n, dtype=torch.int32, device=self.device)
        counts = torch.empty(2, dtype=torch.int64, device=self.device)
        scratch = torch.empty(max(1, B.lib().cuart_route_scratch_bytes(n, 2)), dtype=torch.uint8, device=self.device)
        k, _, keep = B.make_keys((keys, lens) if lens is not None else keys)
        stream = torch.cuda.current_stream(self.device).cuda_stream
        rc = B.lib().cuart_partition_by_flag(B.ctypes.byref(k), n, flags.data_ptr(),
                                             values.data_ptr() if values is not None else None, ok.data_ptr(),
                                             ol.data_ptr() if ol is not None else None,
                                             ov.data_ptr() if ov is not None else None, perm.data_ptr(),
                                             counts.data_ptr(), scratch.data_ptr(), stream)
        B._check(rc, "cuart_partition_by_flag")
        return ok, ol, ov, perm, counts

    def unroute(self, res, perm):
        out = torch.empty_like(res)
        stream = torch.cuda.current_stream(self.device).cuda_stream
        B._check(B.lib().cuart_unroute(res.data_ptr(), perm.data_ptr(), res.shape[0], out.data_ptr(), stream),
                 "cuart_unroute")
        return out

    def lookup(self, index, keys, lens):
        out = torch.empty(keys.shape[0], dtype=torch.int64, device=self.device)
        index.lookup((keys, lens) if lens is not None else keys, out)
        return out

    def update(self, index, keys, lens, values):
        index.update((keys, lens) if lens is not None else keys, values)

    def close(self, index):
        index.close()


# ------------------------------------------------------------------ the protocol
class DistIndex:
    """A CuART index spread over the ranks of a process group."""

    def __init__(self, keys, values, mode="range", group=None, ops=None, lut_bytes=3, splitters=None, local=False,
                 transport="nccl"):
        """keys/values: the GLOBAL key set, identical on every rank (host arrays).
        Range mode keeps this rank's share; replica mode keeps everything.
        local=True: keys/values are already this rank's share of a range partition
        defined by `splitters` (used when the global set is too large to replicate).
        transport: "nccl" (route + all-to-all) or "p2p" (fused push / return over
        peer memory; CUDA ops only)."""
        if mode not in ("range", "replica"):
            raise ValueError(mode)
        if transport not in ("nccl", "p2p"):
            raise ValueError(transport)
        self.mode = mode
        self.transport = transport
        self.windows = None
        self.group = group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        self.ops = ops
        values = np.asarray(values, np.uint64)
        self.kind_bytes = isinstance(keys, tuple)
        if mode == "range":
            if local:
                if splitters is None:
                    raise ValueError("local=True needs the partition's splitters")
                self.splitters_np = np.asarray(splitters, np.uint64)
            else:
                pre = prefix8(keys)
                self.splitters_np = compute_splitters(pre, self.world) if splitters is None else np.asarray(splitters, np.uint64)
                mine = owners(pre, self.splitters_np) == self.rank
                keys, values = select(keys, mine), values[mine]
            self.splitters = ops.tensor(self.splitters_np.view(np.int64).copy()) if self.world > 1 else None
        self.n_local_keys = int(values.shape[0])
        self.index = ops.build(keys, values, lut_bytes)

    # ---- helpers
    # Collectives.  NCCL moves CUDA tensors directly (the product path on the GPU
    # box).  gloo cannot, so CUDA tensors are staged through host memory — this lets
    # the complete GPU path (CuART kernels + this protocol) run as several processes
    # sharing one GPU in tests, where NCCL refuses duplicate devices.
    def _staged(self, t):
        return t.is_cuda and dist.get_backend(self.group) != "nccl"

    def _a2a(self, out, inp, out_splits, in_splits):
        if self._staged(inp):
            ho = out.new_empty(out.shape, device="cpu")
            dist.all_to_all_single(ho, inp.cpu(), out_splits, in_splits, group=self.group)
            out.copy_(ho)
            return
        dist.all_to_all_single(out, inp, out_splits, in_splits, group=self.group)

    def _exchange_counts(self, counts):
        recv = torch.empty_like(counts)
        self._a2a(recv, counts, None, None)
        return recv

    def _split_keys(self, q):
        return (q[0], q[1]) if isinstance(q, tuple) else (q, None)

    # ---- fused p2p transport (range mode)
    def _p2p_route(self, keys, lens, vals):
        """Count, agree on the count matrix, push every op into its owner's window.
        Returns (plan, perm)."""
        n = keys.shape[0]
        kind = B.KIND_BYTES if lens is not None else (B.KIND_U64 if keys.element_size() == 8 else B.KIND_U32)
        ks = B.raw_keys(kind, keys.data_ptr(), lens.data_ptr() if lens is not None else None)
        counts = torch.zeros(self.world, dtype=torch.int64, device=keys.device)
        scratch = torch.empty(max(1, B.lib().cuart_route_scratch_bytes(n, self.world)), dtype=torch.uint8,
                              device=keys.device)
        B.route_count(ks, n, self.splitters.data_ptr(), self.world, counts.data_ptr(), scratch.data_ptr())
        torch.cuda.current_stream(keys.device).synchronize()        # this rank's earlier work on the windows is done
        allc = [torch.empty_like(counts) for _ in range(self.world)]
        if self._staged(counts):
            hc = [torch.empty_like(counts, device="cpu") for _ in range(self.world)]
            dist.all_gather(hc, counts.cpu(), group=self.group)
            allc = hc
        else:
            dist.all_gather(allc, counts, group=self.group)
        M = np.stack([c.cpu().numpy() for c in allc])                 # every rank passed its sync point
        plan = p2p_plan(M, self.rank)
        if self.windows is None:
            self.windows = P2PWindows(self.group, self.world, self.rank, ks_bytes(kind), lens is not None)
        self.windows.ensure(plan["need_recv"], plan["need_res"])
        W, kb = self.windows.peer, self.windows.kb
        perm = torch.empty(n, dtype=torch.int32, device=keys.device)
        B.route_push(ks, n, self.world, vals.data_ptr() if vals is not None else None,
                     [W[o]["keys"] + plan["push_off"][o] * kb for o in range(self.world)],
                     [W[o]["lens"] + plan["push_off"][o] for o in range(self.world)] if lens is not None else None,
                     [W[o]["vals"] + plan["push_off"][o] * 8 for o in range(self.world)] if vals is not None else None,
                     perm.data_ptr(), scratch.data_ptr())
        self._p2p_fence(keys.device)
        return plan, perm, kind

    def _p2p_fence(self, device):
        """Every rank's pushes / returns have landed (kernel completion + barrier)."""
        torch.cuda.current_stream(device).synchronize()
        dist.barrier(group=self.group)

    def _lookup_p2p(self, keys, lens, events=None):
        plan, perm, kind = self._p2p_route(keys, lens, None)
        W, me = self.windows.peer, self.rank
        nr = plan["recv_total"]
        if events:
            events[0].record()
        if nr:
            rk = B.raw_keys(kind, W[me]["keys"], W[me].get("lens"))
            B.lookup_segmented(self.index.h, rk, nr, plan["seg_start"],
                               [W[s]["res"] + plan["res_off"][s] * 8 for s in range(self.world)])
        if events:
            events[1].record()
        self.last_local_lookups = nr
        self._p2p_fence(keys.device)
        out = torch.empty(keys.shape[0], dtype=torch.int64, device=keys.device)
        B.unroute_raw(W[me]["res"], perm.data_ptr(), keys.shape[0], out.data_ptr())
        return out

    def _update_p2p(self, keys, lens, vals):
        plan, _, kind = self._p2p_route(keys, lens, vals)
        W, me = self.windows.peer, self.rank
        nr = plan["recv_total"]
        if nr:
            B.update_raw(self.index.h, B.raw_keys(kind, W[me]["keys"], W[me].get("lens")), nr, W[me]["vals"])

    # ---- lookups
    def lookup(self, queries, events=None):
        """events: optional (start, end) CUDA events recorded around the local lookup kernel."""
        keys, lens = self._split_keys(queries)
        if self.mode == "range" and self.world > 1 and self.transport == "p2p":
            return self._lookup_p2p(keys, lens, events)
        if self.mode == "replica" or self.world == 1:
            if events:
                events[0].record()
            r = self.ops.lookup(self.index, keys, lens)
            if events:
                events[1].record()
            return r
        sk, sl, _, perm, counts = self.ops.route(keys, lens, None, self.splitters, self.world)
        rcounts = self._exchange_counts(counts)
        cs, rs = counts.tolist(), rcounts.tolist()
        rk = sk.new_empty((sum(rs),) + tuple(sk.shape[1:]))
        self._a2a(rk, sk, rs, cs)
        rl = None
        if sl is not None:
            rl = sl.new_empty(sum(rs))
            self._a2a(rl, sl, rs, cs)
        if events:
            events[0].record()
        res = self.ops.lookup(self.index, rk, rl)
        if events:
            events[1].record()
        self.last_local_lookups = int(rk.shape[0])
        back = res.new_empty(keys.shape[0])
        self._a2a(back, res, cs, rs)
        return self.ops.unroute(back, perm)

    # ---- updates (one batch per rank; global order = rank-major)
    def update(self, keys_vals):
        (keys, lens), vals = self._split_keys(keys_vals[0]), keys_vals[1]
        if self.world == 1:
            self.ops.update(self.index, keys, lens, vals)
            return
        if self.mode == "replica":
            gk, gl, gv = self._all_gather_var(keys), (self._all_gather_var(lens) if lens is not None else None), \
                self._all_gather_var(vals)
            self.ops.update(self.index, gk, gl, gv)
            return
        if self.transport == "p2p":
            self._update_p2p(keys, lens, vals)
            return
        sk, sl, sv, _, counts = self.ops.route(keys, lens, vals, self.splitters, self.world)
        rcounts = self._exchange_counts(counts)
        cs, rs = counts.tolist(), rcounts.tolist()
        rk = sk.new_empty((sum(rs),) + tuple(sk.shape[1:]))
        self._a2a(rk, sk, rs, cs)
        rv = sv.new_empty(sum(rs))
        self._a2a(rv, sv, rs, cs)
        rl = None
        if sl is not None:
            rl = sl.new_empty(sum(rs))
            self._a2a(rl, sl, rs, cs)
        self.ops.update(self.index, rk, rl, rv)

    # ---- mixed rounds (config 5, reading C7)
    def mixed_round(self, keys, values, is_update, lens=None, events=None):
        """One round of a mixed op stream: this rank's contiguous slice of the round.
        Every lookup of the round sees the state before the round's updates; the
        updates then apply in global (rank-major, op) order.  Returns per op the
        lookup result, CUART_MISS for update ops."""
        pk, pl, pv, perm, counts = self.ops.partition(keys, lens, values, is_update)
        n_l, n_u = [int(x) for x in counts.tolist()]
        q = (pk[:n_l], pl[:n_l]) if pl is not None else pk[:n_l]
        res = self.lookup(q, events=events)
        uk = (pk[n_l:], pl[n_l:]) if pl is not None else pk[n_l:]
        self.update((uk, pv[n_l:]))
        full = torch.cat([res, res.new_full((n_u,), -1)])
        return self.ops.unroute(full, perm)

    def _all_gather_var(self, t):
        if self._staged(t):
            return self._all_gather_var(t.cpu()).to(t.device)
        n = torch.tensor([t.shape[0]], dtype=torch.int64, device=t.device)
        ns = [torch.empty_like(n) for _ in range(self.world)]
        dist.all_gather(ns, n, group=self.group)
        sizes = [int(x.item()) for x in ns]
        m = max(sizes)
        pad = t.new_zeros((m,) + tuple(t.shape[1:]))
        pad[: t.shape[0]] = t
        g = t.new_empty((self.world * m,) + tuple(t.shape[1:]))
        dist.all_gather_into_tensor(g, pad, group=self.group)
        return torch.cat([g[r * m: r * m + sizes[r]] for r in range(self.world)])

    def close(self):
        if self.windows is not None:
            torch.cuda.synchronize()
            dist.barrier(group=self.group)        # no peer still writes into our windows
            self.windows.close()
            self.windows = None
        if self.index is not None:
            self.ops.close(self.index)
            self.index = None
