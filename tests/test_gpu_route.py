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


@pytest.mark.parametrize("pb", [0, 1])
@pytest.mark.parametrize("kind", ["u64", "u32", "bytes"])
@pytest.mark.parametrize("nparts", [2, 4, 8])
def test_p2p_fused_exchange_loopback(kind, nparts, pb):
    """The fused p2p exchange with P virtual ranks on one GPU: every 'rank' has its
    own partition index and windows (plain device buffers stand in for the mapped
    peer windows), cuart_route_count -> count matrix -> cuart_route_push into the
    owners' windows -> cuart_lookup_segmented straight into the sources' result
    windows -> cuart_unroute.  Then a routed update batch (values pushed with the
    keys, applied in rank-major order).  Results equal the oracle.  pb = 1: the owners'
    indexes pre-bucket every batch of >= 4096 ops (and walk the wide root table), so
    the segmented lookup's last kernel is the bucketed gather storing straight into
    the sources' windows (k_bgather<SEG>)."""
    from paper_conf_icpp_koppehelggp21_b200 import _binding as B
    from paper_conf_icpp_koppehelggp21_b200.dist import p2p_plan, ks_bytes
    rng = np.random.default_rng(nparts * 7 + len(kind))
    if kind == "u64":
        keys = np.unique(rng.integers(0, 2**64, 1 << 16, dtype=np.uint64))
        mkq = lambda m: np.where(rng.random(m) < 0.5, keys[rng.integers(0, keys.shape[0], m)],
                                 rng.integers(0, 2**64, m, dtype=np.uint64))
        bk = B.KIND_U64
    elif kind == "u32":
        keys = np.unique(rng.integers(0, 1 << 24, 1 << 15, dtype=np.uint32))
        mkq = lambda m: rng.integers(0, 1 << 24, m, dtype=np.uint32)
        bk = B.KIND_U32
    else:
        keys = W.string_keys(5, 1 << 14)
        mkq = lambda m: (lambda idx: (keys[0][idx].copy(), keys[1][idx].copy()))(rng.integers(0, 1 << 14, m))
        bk = B.KIND_BYTES
    nk = keys[1].shape[0] if isinstance(keys, tuple) else keys.shape[0]
    vals = rng.integers(0, 2**63, nk, dtype=np.uint64)
    sp = compute_splitters(prefix8(keys), nparts)
    own = owners(prefix8(keys), sp)
    sel = lambda a, m: (a[0][m], a[1][m]) if isinstance(a, tuple) else a[m]
    opt = dict(prebucket=C.PREBUCKET_ON, wide_lut=C.WIDE_ON) if pb else {}
    idx = [C.Index(sel(keys, own == o), vals[own == o], lut_bytes=0 if kind == "bytes" else 3, **opt)
           for o in range(nparts)]
    spt = _t(sp)
    kb = ks_bytes(bk)
    nq = [5000 + 3001 * s for s in range(nparts)]                   # ragged batch per source
    qs = [mkq(m) for m in nq]
    uks = [sel(keys, rng.integers(0, nk, m)) for m in nq]
    uvs = [rng.integers(0, 2**63, m, dtype=np.uint64) for m in nq]

    def raw(a):
        t = _t(a)
        k, l = (t if isinstance(t, tuple) else (t, None))
        return t, B.raw_keys(bk, k.data_ptr(), l.data_ptr() if l is not None else None)

    def exchange(batches, values):
        keep = [raw(b) for b in batches]
        vt = [_t(v) for v in values] if values is not None else None
        scr = [torch.empty(B.lib().cuart_route_scratch_bytes(n, nparts), dtype=torch.uint8, device=DEV) for n in nq]
        cnt = [torch.zeros(nparts, dtype=torch.int64, device=DEV) for _ in nq]
        for s in range(nparts):
            B.route_count(keep[s][1], nq[s], spt.data_ptr(), nparts, cnt[s].data_ptr(), scr[s].data_ptr())
        M = np.stack([c.cpu().numpy() for c in cnt])
        plans = [p2p_plan(M, r) for r in range(nparts)]
        cap = max(plans[0]["need_recv"], 1)
        win = [{"keys": torch.empty(cap * kb, dtype=torch.uint8, device=DEV),
                "lens": torch.empty(cap, dtype=torch.uint8, device=DEV),
                "vals": torch.empty(cap, dtype=torch.int64, device=DEV),
                "res": torch.full((max(plans[0]["need_res"], 1),), 7, dtype=torch.int64, device=DEV)} for _ in nq]
        perms = [torch.empty(n, dtype=torch.int32, device=DEV) for n in nq]
        for s in range(nparts):
            B.route_push(keep[s][1], nq[s], nparts, vt[s].data_ptr() if vt else None,
                         [win[o]["keys"].data_ptr() + plans[s]["push_off"][o] * kb for o in range(nparts)],
                         [win[o]["lens"].data_ptr() + plans[s]["push_off"][o] for o in range(nparts)]
                         if kind == "bytes" else None,
                         [win[o]["vals"].data_ptr() + plans[s]["push_off"][o] * 8 for o in range(nparts)] if vt else None,
                         perms[s].data_ptr(), scr[s].data_ptr())
        torch.cuda.synchronize()
        return plans, win, perms

    plans, win, perms = exchange(qs, None)
    for o in range(nparts):
        p = plans[o]
        if p["recv_total"]:
            rk = B.raw_keys(bk, win[o]["keys"].data_ptr(), win[o]["lens"].data_ptr())
            B.lookup_segmented(idx[o].h, rk, p["recv_total"], p["seg_start"],
                               [win[s]["res"].data_ptr() + p["res_off"][s] * 8 for s in range(nparts)])
    torch.cuda.synchronize()
    mp_ = MapOracle(keys, vals)
    for s in range(nparts):
        out = torch.empty(nq[s], dtype=torch.int64, device=DEV)
        B.unroute_raw(win[s]["res"].data_ptr(), perms[s].data_ptr(), nq[s], out.data_ptr())
        torch.cuda.synchronize()
        assert np.array_equal(out.cpu().numpy().view(np.uint64), mp_.lookup(qs[s])), s
    # routed update batch: values travel with the keys, owners apply in rank-major order
    plans, win, _ = exchange(uks, uvs)
    for o in range(nparts):
        p = plans[o]
        if p["recv_total"]:
            rk = B.raw_keys(bk, win[o]["keys"].data_ptr(), win[o]["lens"].data_ptr())
            B.update_raw(idx[o].h, rk, p["recv_total"], win[o]["vals"].data_ptr())
    torch.cuda.synchronize()
    for s in range(nparts):
        mp_.update(uks[s], uvs[s])
    exp = mp_.lookup(keys)
    got = np.empty(nk, np.uint64)
    for o in range(nparts):
        m = own == o
        out = torch.empty(int(m.sum()), dtype=torch.int64, device=DEV)
        idx[o].lookup(_t(sel(keys, m)), out)
        got[m] = out.cpu().numpy().view(np.uint64)
    assert np.array_equal(got, exp)
    for ix in idx:
        ix.close()
