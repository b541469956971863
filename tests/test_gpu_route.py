"""GPU tests of the multi-GPU routing kernels (cuart_route / cuart_unroute) and a
single-GPU loopback of the range-partitioned path: P partitions' indexes live on
one device and the all-to-all is replaced by slicing the routed runs (SURVEY §4
test-plan item 5).  Results must equal the oracle bit for bit."""
import numpy as np
import pytest
import torch

import paper_conf_icpp_koppehelggp21_b200 as C
from paper_conf_icpp_koppehelggp21_b200.dist import CudaOps, compute_splitters, owners, prefix8
import workloads as W
from oracle import ArtOracle, MapOracle

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


def _np_route(keys, splitters, nparts):
    own = owners(prefix8(keys), splitters)
    order = np.argsort(own, kind="stable")
    perm = np.empty(order.shape[0], np.int64)
    perm[order] = np.arange(order.shape[0])
    return order, perm, np.bincount(own, minlength=nparts)


@pytest.mark.parametrize("kind", ["u64", "u32", "bytes"])
@pytest.mark.parametrize("nparts", [1, 2, 3, 8, 64])
@pytest.mark.parametrize("n", [0, 1, 4095, 4097, 300_001])
def test_route_matches_stable_partition(kind, nparts, n):
    rng = np.random.default_rng(n + nparts)
    if kind == "u64":
        keys = rng.integers(0, 2**64, n, dtype=np.uint64)
    elif kind == "u32":
        keys = rng.integers(0, 2**32, n, dtype=np.uint32)
    else:
        slots = rng.integers(0, 4, (n, 32), dtype=np.uint8)
        lens = rng.integers(1, 33, n).astype(np.uint8)
        keys = (slots, lens)
    vals = rng.integers(0, 2**63, n, dtype=np.uint64)
    sp = compute_splitters(prefix8(keys), nparts)
    ops = CudaOps(DEV)
    kt = _t(keys)
    k, l = (kt if isinstance(kt, tuple) else (kt, None))
    sk, sl, sv, perm, counts = ops.route(k, l, _t(vals), _t(sp) if nparts > 1 else None, nparts)
    torch.cuda.synchronize()
    order, eperm, ecounts = _np_route(keys, sp, nparts)
    assert counts.cpu().numpy().tolist() == ecounts.tolist()
    assert np.array_equal(perm.cpu().numpy().astype(np.int64), eperm)
    if kind == "bytes":
        assert np.array_equal(sk.cpu().numpy(), keys[0][order]) and np.array_equal(sl.cpu().numpy(), keys[1][order])
    else:
        assert np.array_equal(sk.cpu().numpy().view(keys.dtype), keys[order])
    assert np.array_equal(sv.cpu().numpy().view(np.uint64), vals[order])
    back = ops.unroute(sv, perm)
    assert np.array_equal(back.cpu().numpy().view(np.uint64), vals)


@pytest.mark.parametrize("nparts", [2, 4, 8])
def test_loopback_range_partitioned_c1(nparts):
    """Range-partitioned lookups + updates with the CuART kernels, P partitions on one GPU."""
    cfg = W.CONFIGS["c1"]
    keys, vals = W.build_set(cfg)
    pre = prefix8(keys)
    sp = compute_splitters(pre, nparts)
    own = owners(pre, sp)
    parts = [C.Index(keys[own == p], vals[own == p], lut_bytes=3, device=0) for p in range(nparts)]
    ops = CudaOps(DEV)
    spt = _t(sp)

    def routed(qk, qv=None):
        sk, _, sv, perm, counts = ops.route(qk, None, qv, spt, nparts)
        c = counts.cpu().tolist()
        offs = np.concatenate([[0], np.cumsum(c)])
        return sk, sv, perm, offs

    q = W.lookup_batch(cfg, keys, 0, 1 << 18)
    sk, _, perm, offs = routed(_t(q))
    res = torch.empty_like(sk)
    for p in range(nparts):
        if offs[p + 1] > offs[p]:
            parts[p].lookup(sk[offs[p]: offs[p + 1]], res[offs[p]: offs[p + 1]])
    out = ops.unroute(res, perm)
    o = ArtOracle(keys, vals)
    assert np.array_equal(out.cpu().numpy().view(np.uint64), o.lookup(q))
    uk, uv = W.update_batch(cfg, keys)
    sk, sv, _, offs = routed(_t(uk), _t(uv))
    for p in range(nparts):
        if offs[p + 1] > offs[p]:
            parts[p].update(sk[offs[p]: offs[p + 1]], sv[offs[p]: offs[p + 1]])
    o.update(uk, uv)
    sk, _, perm, offs = routed(_t(keys))
    res = torch.empty_like(sk)
    for p in range(nparts):
        parts[p].lookup(sk[offs[p]: offs[p + 1]], res[offs[p]: offs[p + 1]])
    out = ops.unroute(res, perm)
    assert np.array_equal(out.cpu().numpy().view(np.uint64), o.lookup(keys))
    for ix in parts:
        ix.close()
