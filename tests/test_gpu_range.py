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


def test_range_bounds_byte_strings():
    """Byte-string range queries (each leaf class buffer is lexicographically
    ordered): per class c, start = #class-c keys < lo and end = #class-c keys <= hi in
    true byte-string order (a proper prefix sorts first), against Python's bytes
    ordering over the key set.  Bounds include exact keys, proper prefixes of keys
    (the zero-padded bytes agree, the length decides), keys with a bumped last byte,
    random strings, and empty ranges."""
    import bisect
    slots, lens = W.string_keys(4, 50_000, min_len=2)
    keys = [bytes(slots[i, : lens[i]]) for i in range(lens.shape[0])]
    vals = np.arange(lens.shape[0], dtype=np.uint64)
    ix = C.Index((slots, lens), vals)
    rng = np.random.default_rng(9)
    m = 20_000
    pick = rng.integers(0, len(keys), m)
    lo_b, hi_b = [], []
    for j, p in enumerate(pick):
        k = keys[p]
        r = j % 5
        if r == 0:
            a, b = k, k                                                # exactly one key
        elif r == 1:
            a, b = k[: max(1, len(k) // 2)], k                         # a proper prefix as the lower bound
        elif r == 2:
            a = k[:-1] + bytes([min(255, k[-1] + 1)])
            b = keys[pick[(j + 1) % m]]
        elif r == 3:
            a = bytes(rng.integers(97, 123, rng.integers(1, 33)).astype(np.uint8))
            b = bytes(rng.integers(97, 123, rng.integers(1, 33)).astype(np.uint8))
        else:
            a, b = k, k[: max(1, len(k) - 3)]                          # hi < lo: empty
        lo_b.append(a)
        hi_b.append(b)

    def pack(xs):
        s_ = np.zeros((len(xs), 32), np.uint8)
        l_ = np.zeros(len(xs), np.uint8)
        for i, x in enumerate(xs):
            s_[i, : len(x)] = np.frombuffer(x, np.uint8)
            l_[i] = len(x)
        return torch.from_numpy(s_).to(DEV), torch.from_numpy(l_).to(DEV)

    b = ix.range(pack(lo_b), pack(hi_b))
    torch.cuda.synchronize()
    b = b.cpu().numpy()
    classes = [sorted(k for k in keys if len(k) <= 8), sorted(k for k in keys if 8 < len(k) <= 16),
               sorted(k for k in keys if len(k) > 16)]
    assert all(len(c) > 0 for c in classes)
    for i in range(m):
        for c, ks in enumerate(classes):
            s = bisect.bisect_left(ks, lo_b[i])
            e = max(s, bisect.bisect_right(ks, hi_b[i]))
            assert (b[i, 2 * c], b[i, 2 * c + 1]) == (s, e), (i, c, lo_b[i], hi_b[i])
    # the leaf records of each class are that class's keys in this order
    view = ix.dump()
    for c, (t, w) in enumerate(((5, 8), (6, 16), (7, 32))):
        rec = view["buf"][t].reshape(-1, int(view["record_bytes"][t]))[:, :w]
        assert [bytes(r).rstrip(b"\0") for r in rec[:200]] == [k.rstrip(b"\0") for k in classes[c][:200]]
    ix.close()
