"""GPU parity of the byte-string skip table (cuart_build_opts.skip_log2):
a walk that starts at the node covering the query's first D bytes must return what
the plain-map oracle returns -- for every table size (D small, the library's choice,
D = 16), for queries shorter than D, queries whose D-byte prefix no key has, hits of
every key class, after update batches (the update walk starts from the table too)
and after deletes (tombstones behind table entries read as absent)."""
import numpy as np
import pytest
import torch

import paper_conf_icpp_koppehelggp21_b200 as C
import workloads as W
from oracle import MapOracle

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda:0")


def _dev(batch):
    slots, lens = batch
    return (torch.from_numpy(np.ascontiguousarray(slots)).to(DEV), torch.from_numpy(np.ascontiguousarray(lens)).to(DEV))


def _lookup(ix, batch):
    q = _dev(batch)
    out = torch.empty(q[1].shape[0], dtype=torch.int64, device=DEV)
    ix.lookup(q, out)
    torch.cuda.synchronize()
    return out.cpu().numpy().view(np.uint64)


def _queries(keys, rng, m):
    slots, lens = keys
    n = lens.shape[0]
    hit = rng.integers(0, n, m)
    qs, ql = slots[hit].copy(), lens[hit].copy()
    # a third: perturb one byte inside or past the first 16 (absent prefixes / absent keys)
    pert = rng.random(m) < 0.33
    pos = rng.integers(0, 32, m)
    pos = np.minimum(pos, np.maximum(ql.astype(np.int64) - 2, 0))
    qs[pert, pos[pert]] = (qs[pert, pos[pert]].astype(np.int64) % 250 + 1 + rng.integers(0, 4, pert.sum())).astype(np.uint8)
    # some short queries (length < D): prefixes of keys, zero-padded
    short = rng.random(m) < 0.1
    nl = rng.integers(1, 9, m).astype(np.uint8)
    ql = np.where(short, np.minimum(ql, nl), ql).astype(np.uint8)
    idx = np.arange(32)[None, :] >= ql[:, None]
    qs[idx] = 0
    return qs, ql


@pytest.mark.parametrize("skip_log2", [12, 0, 26])
def test_skip_table_lookups_updates_deletes(skip_log2):
    rng = np.random.default_rng(skip_log2 + 5)
    keys = W.string_keys(4, 1 << 17)
    n = keys[1].shape[0]
    vals = rng.integers(0, 2**63, n, dtype=np.uint64)
    ix = C.Index(keys, vals, lut_bytes=3, skip_log2=skip_log2)
    st = ix.stats()
    assert st["skip_prefix"] > 3 and st["skip_slots"] > 0, st
    if skip_log2 == 26:
        assert st["skip_prefix"] == 16
    mp = MapOracle(keys, vals)
    q = _queries(keys, rng, 150_001)
    assert np.array_equal(_lookup(ix, q), mp.lookup(q))
    # updates through the table (duplicates: the highest op index wins)
    pick = rng.integers(0, n, 40_000)
    uk = (keys[0][pick].copy(), keys[1][pick].copy())
    uv = rng.integers(0, 2**63, pick.shape[0], dtype=np.uint64)
    ix.update(_dev(uk), torch.from_numpy(uv.view(np.int64)).to(DEV))
    mp.update(uk, uv)
    assert np.array_equal(_lookup(ix, keys), mp.lookup(keys))
    # deletes (non-structural, tombstones) then lookups through the table
    dk = keys[0][:5000].copy(), keys[1][:5000].copy()
    ix.erase(_dev(dk))
    mp.apply(dk, np.zeros(5000, np.uint64), np.ones(5000, dtype=bool))
    assert np.array_equal(_lookup(ix, keys), mp.lookup(keys))
    assert np.array_equal(_lookup(ix, q), mp.lookup(q))
    assert ix.get_error() == 0
    ix.close()


def test_skip_table_disabled_equals_enabled(monkeypatch):
    """CUART_SKIP=0 (no table) and the default table give identical results on a
    c4-shaped Zipf batch."""
    keys = W.string_keys(4, 1 << 16)
    vals = np.arange(1 << 16, dtype=np.uint64) + 3
    q = (lambda idx: (keys[0][idx].copy(), keys[1][idx].copy()))(
        W.string_lookup_at(W.CONFIGS["c4"], 1 << 16, np.arange(300_000)))
    on = C.Index(keys, vals, lut_bytes=3)
    monkeypatch.setenv("CUART_SKIP", "0")
    off = C.Index(keys, vals, lut_bytes=3)
    assert off.stats()["skip_prefix"] == 0 and on.stats()["skip_prefix"] > 0
    assert np.array_equal(_lookup(on, q), _lookup(off, q))
    on.close()
    off.close()
