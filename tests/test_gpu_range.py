"""GPU range queries (§8(f) f2): (start, end) leaf indices of [lo, hi]
against the plain definition: positions in the lexicographically sorted key set
(the oracle's in-order dump)."""
import numpy as np
import pytest
import torch

import paper_conf_icpp_koppehelggp21_b200 as C
import workloads as W
from oracle import ArtOracle

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda:0")


def _t(a):
    if a.dtype == np.uint64:
        return torch.from_numpy(a.view(np.int64)).to(DEV)
    return torch.from_numpy(a.view(np.int32)).to(DEV)


def _sorted_keys(keys, kind):
    ks, ls, _ = ArtOracle(keys, np.zeros(keys.shape[0], np.uint64)).dump_inorder()
    L = 8 if kind == "u64" else 4
    return np.ascontiguousarray(ks[:, :L]).view(">u8" if L == 8 else ">u4").ravel().astype(
        np.uint64 if L == 8 else np.uint32)


@pytest.mark.parametrize("kind", ["u64", "u32"])
def test_range_bounds(kind):
    rng = np.random.default_rng(3)
    if kind == "u64":
        keys, _ = W.build_set(W.CONFIGS["c1"])
        lo = rng.integers(0, 2**64, 100_000, dtype=np.uint64)
        span = rng.integers(0, 2**58, 100_000, dtype=np.uint64)
        hi = lo + span
        hi[hi < lo] = np.uint64(2**64 - 1)
        lo[:1000] = keys[:1000]                       # exact-key bounds (inclusive at both ends)
        hi[:1000] = keys[:1000]
        lo[1000:1010] = 0
        hi[1000:1010] = np.uint64(2**64 - 1)
    else:
        keys = (np.arange(1 << 16, dtype=np.uint32) * 7919) & np.uint32(0xFFFFFF)
        keys = np.unique(keys)
        lo = rng.integers(0, 2**24, 100_000, dtype=np.uint32)
        hi = (lo + rng.integers(0, 5000, 100_000, dtype=np.uint32)).astype(np.uint32)
        hi[:10] = lo[:10] - np.uint32(1)               # empty ranges (hi < lo)
    vals = np.arange(keys.shape[0], dtype=np.uint64)
    ix = C.Index(keys, vals)
    b = ix.range(_t(lo), _t(hi))
    torch.cuda.synchronize()
    b = b.cpu().numpy()
    sk = _sorted_keys(keys, kind)
    s = np.searchsorted(sk, lo, side="left")
    e = np.maximum(np.searchsorted(sk, hi, side="right"), s)
    assert np.array_equal(b[:, 0], s) and np.array_equal(b[:, 1], e)
    assert not b[:, 2:].any()
    # the leaves [start, end) of the leaf8 buffer are exactly the keys in range
    view = ix.dump()
    leaf_keys = view["buf"][5].reshape(-1, int(view["record_bytes"][5]))[:, :8].copy()
    if kind == "u64":
        lk = leaf_keys.view(">u8").ravel().astype(np.uint64)
    else:
        lk = np.ascontiguousarray(leaf_keys[:, :4]).view(">u4").ravel().astype(np.uint32)
    assert np.array_equal(lk, sk)
    ix.close()


def test_range_with_deletes_keeps_positions():
    keys = np.arange(0, 1000, 10, dtype=np.uint64)
    ix = C.Index(keys, keys + np.uint64(1))
    ix.erase(_t(keys[10:20]))
    b = ix.range(_t(np.array([0, 95, 150], np.uint64)), _t(np.array([999, 200, 150], np.uint64)))
    torch.cuda.synchronize()
    assert b.cpu().numpy()[:, :2].tolist() == [[0, 100], [10, 21], [15, 16]]
    dv = ix.dump()
    leaves = dv["buf"][5].reshape(-1, int(dv["record_bytes"][5]))
    vals = leaves[:, 8:16].copy().view(np.uint64).ravel()
    assert np.all(vals[10:20] == np.uint64(2**64 - 1)) and vals[20] == 201   # tombstones in place
    ix.close()
