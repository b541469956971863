"""GPU parity of non-structural device deletes (§8(f) f1) and mixed
update/delete batches (reading C17) against the CPU oracle."""
import random

import numpy as np
import pytest
import torch

import paper_conf_icpp_koppehelggp21_b200 as C
import workloads as W
from oracle import ArtOracle, MapOracle, OART_MISS
from tests.layout_decode import to_records

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda:0")
MISS = int(OART_MISS)


def _t(a):
    if isinstance(a, tuple):
        return (_t(a[0]), _t(a[1]))
    if a.dtype == np.uint64:
        return torch.from_numpy(a.view(np.int64)).to(DEV)
    if a.dtype == np.uint32:
        return torch.from_numpy(a.view(np.int32)).to(DEV)
    return torch.from_numpy(a).to(DEV)


def _lookup(ix, q):
    qt = _t(q)
    n = (qt[0] if isinstance(qt, tuple) else qt).shape[0]
    out = torch.empty(n, dtype=torch.int64, device=DEV)
    ix.lookup(qt, out)
    torch.cuda.synchronize()
    return out.cpu().numpy().view(np.uint64)


def test_delete_hand_pins_gpu():
    keys = np.array([1 << 40, 2 << 40, 3 << 40, 3 << 40 | 1], np.uint64)
    for lut, fmt in ((0, 1), (3, 1), (3, 2), (3, 3)):
        ix = C.Index(keys, np.array([10, 20, 30, 40], np.uint64), lut_bytes=lut, lut_format=fmt)
        ix.erase(_t(np.array([keys[0], 12345], np.uint64)))
        assert _lookup(ix, keys).tolist() == [MISS, 20, 30, 40]
        ix.update_ex(_t(np.array([keys[1], keys[1]], np.uint64)), _t(np.array([0, 21], np.uint64)),
                     _t(np.array([1, 0], np.uint8)))
        ix.update_ex(_t(np.array([keys[2], keys[2]], np.uint64)), _t(np.array([31, 0], np.uint64)),
                     _t(np.array([0, 1], np.uint8)))
        assert _lookup(ix, keys).tolist() == [MISS, 21, MISS, 40]
        ix.update(_t(np.array([keys[0], keys[2]], np.uint64)), _t(np.array([5, 6], np.uint64)))
        assert _lookup(ix, keys).tolist() == [MISS, 21, MISS, 40]
        assert sorted(ix.free_leaves().tolist()) == [0, 2]      # leaf ids in key order
        assert ix.get_error() == 0
        ix.close()


def test_delete_single_key_root_leaf():
    ix = C.Index(np.array([7], np.uint64), np.array([70], np.uint64), lut_bytes=0)
    ix.erase(_t(np.array([7], np.uint64)))
    assert _lookup(ix, np.array([7, 8], np.uint64)).tolist() == [MISS, MISS]
    ix.update(_t(np.array([7], np.uint64)), _t(np.array([1], np.uint64)))
    assert _lookup(ix, np.array([7], np.uint64)).tolist() == [MISS]
    ix.close()


@pytest.mark.parametrize("kind", ["u64", "bytes"])
@pytest.mark.parametrize("lut,fmt", [(0, 1), (3, 2), (3, 3), (2, 1)])
def test_mixed_batches_vs_oracle(kind, lut, fmt):
    cfg = W.CONFIGS["c1"]
    if kind == "u64":
        keys, vals = W.build_set(cfg)
    else:
        keys = W.string_keys(4, 30_000)
        vals = np.arange(30_000, dtype=np.uint64) * 11 + 3
    n = keys[1].shape[0] if isinstance(keys, tuple) else keys.shape[0]
    o = ArtOracle(keys, vals)
    mp = MapOracle(keys, vals)
    ix = C.Index(keys, vals, lut_bytes=lut, lut_format=fmt)
    rng = np.random.default_rng(lut * 10 + fmt)
    for rnd in range(4):
        m = 50_000
        pick = rng.integers(0, n, m)
        if isinstance(keys, tuple):
            bk = (keys[0][pick].copy(), keys[1][pick].copy())
        else:
            bk = keys[pick].copy()
            bk[rng.random(m) < 0.05] ^= np.uint64(1 << 7)          # some absent keys
        bv = rng.integers(0, 2**63, m, dtype=np.uint64)
        bd = (rng.random(m) < (0.3 if rnd < 3 else 0.9)).astype(np.uint8)
        ix.update_ex(_t(bk), _t(bv), _t(bd))
        o.apply(bk, bv, bd)
        mp.apply(bk, bv, bd)
        exp = mp.lookup(keys)
        assert np.array_equal(o.lookup(keys), exp)
        assert np.array_equal(_lookup(ix, keys), exp), rnd
    # dump after deletes: live structure == oracle (nodes not collapsed; tombstones skipped)
    assert to_records(ix.dump()) == o.dump_structure().tolist()
    deleted = int((mp.lookup(keys) == OART_MISS).sum())
    fl = ix.free_leaves()
    assert fl.shape[0] == deleted and np.unique(fl).shape[0] == deleted
    ix.close()


@pytest.mark.parametrize("fmt", [1, 3])
@pytest.mark.parametrize("wide", [0, 2])
def test_deletes_visible_to_bucketed_wide_walk(fmt, wide):
    """Pre-bucketed lookups start from the wide root table (LUT link + the target
    node's keys).  Deletes unlink leaves from node slots AND from LUT entries (at
    k = 3 most of c1's keys hang directly off a LUT entry); both must be visible to
    the bucketed walk, and bucketed plain updates after the deletes must skip the
    deleted keys (reading C18)."""
    cfg = W.CONFIGS["c1"]
    keys, vals = W.build_set(cfg)
    rng = np.random.default_rng(5)
    # 3-byte prefixes holding 2..16 keys each: LUT entries leading to N4 / N16 nodes
    dense = (np.repeat(np.arange(1 << 12, dtype=np.uint64), 6) << np.uint64(40)) | \
        rng.integers(0, 1 << 40, 6 << 12, dtype=np.uint64) | np.uint64(0xAB << 56)
    keys = np.unique(np.concatenate([keys, dense]))
    vals = rng.integers(0, 2**63, keys.shape[0], dtype=np.uint64)
    on = C.Index(keys, vals, lut_bytes=3, lut_format=fmt, prebucket=C.PREBUCKET_ON, wide_lut=wide)
    mp = MapOracle(keys, vals)
    dk = keys[rng.random(keys.shape[0]) < 0.4]
    on.erase(_t(dk))
    mp.apply(dk, None, np.ones(dk.shape[0], bool))
    q = np.concatenate([keys, rng.integers(0, 2**64, 1 << 16, dtype=np.uint64)])
    assert np.array_equal(_lookup(on, q), mp.lookup(q))
    uk = keys[rng.integers(0, keys.shape[0], 100_000)]
    uv = rng.integers(0, 2**63, uk.shape[0], dtype=np.uint64)
    on.update(_t(uk), _t(uv))
    mp.update(uk, uv)
    assert np.array_equal(_lookup(on, q), mp.lookup(q))
    on.close()


@pytest.mark.parametrize("wide", [0, 2])
def test_deletes_visible_through_full_n256_leaf_run(wide):
    """Dense u32 keys (c2 shape): every 3-byte prefix leads to a full N256 whose 256
    children are consecutive leaves, so the wide root table's leaf run addresses
    the leaf without the N256 child link (kernels.cuh start_wide).  A delete nulls
    that child link; the run still reaches the leaf, whose tombstone (C18) must
    read as absent to lookups and make later updates skip it."""
    rng = np.random.default_rng(11)
    keys = np.arange(1 << 18, dtype=np.uint32)
    vals = rng.integers(0, 2**63, keys.shape[0], dtype=np.uint64)
    on = C.Index(keys, vals, lut_bytes=3, prebucket=C.PREBUCKET_ON, wide_lut=wide)
    mp = MapOracle(keys, vals)
    dk = keys[rng.random(keys.shape[0]) < 0.4]
    on.erase(_t(dk))
    mp.apply(dk, None, np.ones(dk.shape[0], bool))
    q = np.concatenate([keys, rng.integers(0, 2**32, 1 << 16, dtype=np.uint64).astype(np.uint32)])
    assert np.array_equal(_lookup(on, q), mp.lookup(q))
    uk = keys[rng.integers(0, keys.shape[0], 100_000)]
    uv = rng.integers(0, 2**63, uk.shape[0], dtype=np.uint64)
    on.update(_t(uk), _t(uv))
    mp.update(uk, uv)
    assert np.array_equal(_lookup(on, q), mp.lookup(q))
    on.close()
