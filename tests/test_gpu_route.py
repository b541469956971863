"""GPU tests of the stable partition primitive (cuart_route / cuart_unroute, the
kernels behind cuart_partition_by_flag): per-owner runs, stable in op order, and
the inverse permutation, against a numpy stable partition.  The multi-GPU layer
proper (cuart_dist_*) is tested in tests/test_gpu_dist.py."""
import ctypes

import numpy as np
import pytest
import torch

import paper_conf_icpp_koppehelggp21_b200 as C
from paper_conf_icpp_koppehelggp21_b200 import _binding as B
from paper_conf_icpp_koppehelggp21_b200.dist import owners, prefix8

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


def _splitters(prefix, nparts):
    """nparts-1 quantile splitters of the sample (owner = number of splitters <= prefix)."""
    if nparts <= 1:
        return np.zeros(0, np.uint64)
    s = np.sort(prefix)
    if s.shape[0] == 0:
        return np.arange(1, nparts, dtype=np.uint64) * np.uint64((1 << 64) // nparts)
    return s[(np.arange(1, nparts) * s.shape[0]) // nparts].astype(np.uint64)


def _route(keys, lens, values, splitters, nparts):
    n = keys.shape[0]
    send_keys = torch.empty_like(keys)
    send_lens = torch.empty_like(lens) if lens is not None else None
    send_vals = torch.empty_like(values)
    perm = torch.empty(n, dtype=torch.int32, device=DEV)
    counts = torch.empty(nparts, dtype=torch.int64, device=DEV)
    scratch = torch.empty(max(1, B.lib().cuart_route_scratch_bytes(n, nparts)), dtype=torch.uint8, device=DEV)
    k, _, keep = B.make_keys((keys, lens) if lens is not None else keys)
    stream = torch.cuda.current_stream().cuda_stream
    B._check(B.lib().cuart_route(ctypes.byref(k), n, splitters.data_ptr() if nparts > 1 else None, nparts,
                                 values.data_ptr(), send_keys.data_ptr(),
                                 send_lens.data_ptr() if send_lens is not None else None, send_vals.data_ptr(),
                                 perm.data_ptr(), counts.data_ptr(), scratch.data_ptr(), stream), "cuart_route")
    return send_keys, send_lens, send_vals, perm, counts


def _unroute(res, perm):
    out = torch.empty_like(res)
    B._check(B.lib().cuart_unroute(res.data_ptr(), perm.data_ptr(), res.shape[0], out.data_ptr(),
                                   torch.cuda.current_stream().cuda_stream), "cuart_unroute")
    return out


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
    sp = _splitters(prefix8(keys), nparts)
    kt = _t(keys)
    k, l = (kt if isinstance(kt, tuple) else (kt, None))
    sk, sl, sv, perm, counts = _route(k, l, _t(vals), _t(sp) if nparts > 1 else None, nparts)
    torch.cuda.synchronize()
    order, eperm, ecounts = _np_route(keys, sp, nparts)
    assert counts.cpu().numpy().tolist() == ecounts.tolist()
    assert np.array_equal(perm.cpu().numpy().astype(np.int64), eperm)
    if kind == "bytes":
        assert np.array_equal(sk.cpu().numpy(), keys[0][order]) and np.array_equal(sl.cpu().numpy(), keys[1][order])
    else:
        assert np.array_equal(sk.cpu().numpy().view(keys.dtype), keys[order])
    assert np.array_equal(sv.cpu().numpy().view(np.uint64), vals[order])
    back = _unroute(sv, perm)
    assert np.array_equal(back.cpu().numpy().view(np.uint64), vals)


@pytest.mark.parametrize("kind", ["u64", "u32", "bytes"])
@pytest.mark.parametrize("n,p", [(1, 0.5), (4095, 0.1), (4096 * 3 + 17, 0.1), (200_003, 0.5), (70_001, 0.0),
                                 (70_001, 1.0)])
def test_partition_by_flag_matches_stable_partition(kind, n, p):
    """cuart_partition_by_flag (the two-way partition that splits config 5's mixed
    rounds, reading C7): flag-0 ops first, then flag-1 ops, each in op order, with
    the values carried along; perm[i] = slot of op i and cuart_unroute inverts it.
    Ragged tails, all-lookup and all-update batches, and a flags view 1 byte into
    its buffer (unaligned 16-B flag loads fall back to scalar loads)."""
    rng = np.random.default_rng(n + int(p * 10))
    if kind == "u64":
        keys = rng.integers(0, 2**64, n, dtype=np.uint64)
        lens = None
    elif kind == "u32":
        keys = rng.integers(0, 2**32, n, dtype=np.uint32)
        lens = None
    else:
        keys = rng.integers(1, 256, (n, 32), dtype=np.uint8)
        lens = rng.integers(1, 33, n, dtype=np.uint8)
    vals = rng.integers(0, 2**63, n, dtype=np.uint64)
    flags = (rng.random(n) < p).astype(np.uint8)
    order = np.argsort(flags, kind="stable")
    want_perm = np.empty(n, np.int64)
    want_perm[order] = np.arange(n)
    for off in (0, 1):
        fbuf = torch.zeros(n + 1, dtype=torch.uint8, device=DEV)
        fv = fbuf[off:off + n]
        fv.copy_(torch.from_numpy(flags).to(DEV))
        kt = _t(keys)
        lt = _t(lens) if lens is not None else None
        vt = _t(vals)
        ok, ov = torch.empty_like(kt), torch.empty_like(vt)
        ol = torch.empty_like(lt) if lt is not None else None
        perm = torch.empty(n, dtype=torch.int32, device=DEV)
        counts = torch.empty(2, dtype=torch.int64, device=DEV)
        scratch = torch.empty(max(1, B.lib().cuart_route_scratch_bytes(n, 2)), dtype=torch.uint8, device=DEV)
        k, _, keep = B.make_keys((kt, lt) if lt is not None else kt)
        stream = torch.cuda.current_stream().cuda_stream
        B._check(B.lib().cuart_partition_by_flag(ctypes.byref(k), n, fv.data_ptr(), vt.data_ptr(), ok.data_ptr(),
                                                 ol.data_ptr() if ol is not None else None, ov.data_ptr(),
                                                 perm.data_ptr(), counts.data_ptr(), scratch.data_ptr(), stream),
                 "cuart_partition_by_flag")
        torch.cuda.synchronize()
        nl = int((flags == 0).sum())
        assert counts.cpu().tolist() == [nl, n - nl]
        assert np.array_equal(perm.cpu().numpy().astype(np.int64), want_perm)
        got_k = ok.cpu().numpy()
        assert np.array_equal(got_k.view(keys.dtype) if kind != "bytes" else got_k, keys[order])
        if lens is not None:
            assert np.array_equal(ol.cpu().numpy(), lens[order])
        assert np.array_equal(ov.cpu().numpy().view(np.uint64), vals[order])
        back = _unroute(ov, perm)
        assert np.array_equal(back.cpu().numpy().view(np.uint64), vals)
