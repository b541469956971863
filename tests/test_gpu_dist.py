"""The multi-GPU layer (cuart_dist_*, csrc/dist.cu) on one GPU with P virtual ranks:
P threads of this process, each a rank with its own cuart_dist index, stream and
receive windows on cuda:0, the host bootstrap a thread barrier
(dist.ThreadAllGather).  Transport P2P runs its real device protocol: the fused
K-ROUTE/K-BUCKET scatter stores into the owners' windows, device-side release /
acquire flags order the ranks, the owner's walk returns results into the sources'
windows.  (Windows of a virtual rank are used directly; separate processes map
them with CUDA IPC, tests/test_gpu_dist_procs.py.)  Transport NCCL needs one GPU
per rank, so it runs at P = 1 here.

Every result is compared bit for bit with the plain-map oracle: lookups of every
rank's batch, the state after update calls whose batches are applied in
rank-major order (reading C7; duplicates inside a batch, across ranks and across
chunks, reserved values dropped, reading C5), config 5's mixed rounds, with chunks
small enough that every call runs many pipeline chunks."""
import threading

import numpy as np
import pytest
import torch

import workloads as W
from oracle import MapOracle, OART_MISS
from paper_conf_icpp_koppehelggp21_b200.dist import DistIndex, ThreadAllGather

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda:0")


def _t(a):
    if isinstance(a, tuple):
        return (_t(a[0]), _t(a[1]))
    if a.dtype == np.uint64:
        return torch.from_numpy(a.view(np.int64)).to(DEV)
    if a.dtype == np.uint32:
        return torch.from_numpy(a.view(np.int32)).to(DEV)
    return torch.from_numpy(a).to(DEV)


def _u64(t):
    return t.cpu().numpy().view(np.uint64)


def _take(keys, idx):
    return (keys[0][idx], keys[1][idx]) if isinstance(keys, tuple) else keys[idx]


def _keyset(kind, n):
    if kind == "u64":
        return W.u64_keys(7, n)
    if kind == "u32":
        return np.arange(n, dtype=np.uint32) * np.uint32(3)        # dense-ish, common leading bytes
    return W.string_keys(4, n)


def _batches(kind, keys, P, call, sizes):
    """Per-rank batches: mostly present keys (with duplicates), some absent ones."""
    out = []
    n = keys[1].shape[0] if isinstance(keys, tuple) else keys.shape[0]
    for r in range(P):
        rng = np.random.default_rng(1000 * call + r)
        m = sizes[(r + call) % len(sizes)]
        pick = rng.integers(0, n, m)
        k = _take(keys, pick)
        if kind == "u64":
            k = np.where(rng.random(m) < 0.85, k, rng.integers(0, 2**64, m, dtype=np.uint64))
        elif kind == "u32":
            k = np.where(rng.random(m) < 0.85, k, (rng.integers(0, n, m) * 3 + 1).astype(np.uint32))
        v = rng.integers(0, 2**63, m, dtype=np.uint64)
        v[::97] = OART_MISS
        out.append((k, v))
    return out


def _run(P, fn):
    """Run fn(rank, gather) in P threads; re-raise the first failure."""
    g = ThreadAllGather(P)
    res, errs = [None] * P, []

    def work(r):
        try:
            torch.cuda.set_device(DEV)
            s = torch.cuda.Stream(DEV)
            with torch.cuda.stream(s):
                res[r] = fn(r, g.bind(r), s)
        except BaseException as e:  # noqa: BLE001
            errs.append(e)
            g.barrier.abort()

    th = [threading.Thread(target=work, args=(r,)) for r in range(P)]
    for t in th:
        t.start()
    for t in th:
        t.join(600)
    if errs:
        raise errs[0]
    return res


CASES = [(k, m, t, p) for k in ("u64", "u32", "bytes") for m in ("range", "replica")
         for t, p in (("p2p", 1), ("p2p", 2), ("p2p", 3), ("nccl", 1))] + \
        [("u64", "range", "p2p", 8), ("u64", "replica", "p2p", 8), ("bytes", "range", "p2p", 4)]


@pytest.mark.parametrize("kind,mode,transport,P", CASES)
def test_dist_virtual_ranks(kind, mode, transport, P):
    n = 40_000
    keys = _keyset(kind, n)
    vals = W.values_for(W.SEED_VALUES + 7, np.arange(n, dtype=np.uint64))
    chunk = 8192                      # many chunks per call (two window slots in flight)
    calls = [_batches(kind, keys, P, c, [30_000, 0, 11_111, 4097]) for c in range(2)]
    looks = [_batches(kind, keys, P, 10 + c, [25_000, 1, 9_999])[r][0] for c in range(1) for r in range(P)]

    def fn(r, gather, s):
        di = DistIndex(keys, vals, mode=mode, transport=transport, rank=r, world=P, gather=gather, chunk=chunk,
                       lut_bytes=3 if kind != "bytes" else 0)
        out = {"look0": _u64(di.lookup(_t(looks[r]))) if _len(looks[r]) else np.zeros(0, np.uint64)}
        for c, batch in enumerate(calls):
            k, v = batch[r]
            di.update(_t(k), _t(v))
            res = di.lookup(_t(keys))
            s.synchronize()
            out[f"after{c}"] = _u64(res)
        out["recv"] = di.last()
        di.close()
        return out

    res = _run(P, fn)
    o = MapOracle(keys, vals)
    for r in range(P):
        if _len(looks[r]):
            assert np.array_equal(res[r]["look0"], o.lookup(looks[r])), r
    for c, batch in enumerate(calls):
        for r in range(P):                                   # rank-major global order (reading C7)
            o.update(*batch[r])
        exp = o.lookup(keys)
        for r in range(P):
            assert np.array_equal(res[r][f"after{c}"], exp), (c, r)
    if mode == "range":                                     # every key served by exactly one owner
        assert sum(x["recv"][0] for x in res) == P * n


def _len(k):
    return k[1].shape[0] if isinstance(k, tuple) else k.shape[0]


@pytest.mark.parametrize("fused", [True, False])
@pytest.mark.parametrize("P", [1, 2, 4])
def test_dist_mixed_rounds_p_independent(P, fused):
    """Config 5's recipe (reading C7) at 2^16 keys: rounds of mixed ops, rank r
    originating the r-th 1/P slice of each round; outputs equal the single-stream
    oracle replay, so they do not depend on P.  fused: one cuart_dist_mixed call per
    round (filtered passes); else partition + dist lookup + dist update + unroute."""
    n, R, rounds = 1 << 16, 1 << 17, 3
    keys = W.u64_keys(5, n)
    vals = W.values_for(W.SEED_VALUES + 5, np.arange(n, dtype=np.uint64))
    per = R // P

    def fn(r, gather, s):
        di = DistIndex(keys, vals, mode="range", transport="p2p", rank=r, world=P, gather=gather, chunk=1 << 14)
        outs = []
        for rd in range(rounds):
            k, u, v = W.mixed_ops_torch(5, n, rd * R + r * per, per, DEV)
            outs.append(_u64(di.mixed_round(k, v, u, fused=fused)))
        di.close()
        return np.concatenate(outs)

    res = _run(P, fn)
    o = MapOracle(keys, vals)
    for rd in range(rounds):
        k, u, v = W.mixed_ops(5, n, np.arange(rd * R, (rd + 1) * R))
        exp = o.lookup(k)
        exp[u == 1] = OART_MISS
        got = np.concatenate([res[r][rd * per:(rd + 1) * per] for r in range(P)])
        assert np.array_equal(got, exp), rd
        o.update(k[u == 1], v[u == 1])
