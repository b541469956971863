"""Config-5 semantics on one GPU: mixed lookup/update rounds (reading C7) through
the multi-GPU layer at world size 1 (cuart_dist_* with both transports), against
the oracle replay."""
import os

import numpy as np
import pytest
import torch
import torch.distributed as dist

import workloads as W
from oracle import MapOracle, OART_MISS

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda:0")


@pytest.fixture(scope="module")
def pg():
    if not dist.is_initialized():
        store = dist.HashStore()
        dist.init_process_group("gloo", store=store, rank=0, world_size=1)
    yield
    dist.destroy_process_group()


@pytest.mark.parametrize("transport", ["p2p", "nccl"])
def test_mixed_rounds_single_gpu(pg, transport):
    from paper_conf_icpp_koppehelggp21_b200.dist import DistIndex
    n, R, rounds = 1 << 18, 1 << 20, 4
    keys = W.u64_keys(5, n)
    vals = W.values_for(W.SEED_VALUES + 5, np.arange(n, dtype=np.uint64))
    di = DistIndex(keys, vals, mode="range", transport=transport)
    o = MapOracle(keys, vals)
    for r in range(rounds):
        k, u, v = W.mixed_ops_torch(5, n, r * R, R, DEV)
        out = di.mixed_round(k, v, u)
        torch.cuda.synchronize()
        kn, un, vn = W.mixed_ops(5, n, np.arange(r * R, (r + 1) * R))
        assert np.array_equal(k.cpu().numpy().view(np.uint64), kn)
        exp = o.lookup(kn)
        exp[un == 1] = OART_MISS
        assert np.array_equal(out.cpu().numpy().view(np.uint64), exp), r
        o.update(kn[un == 1], vn[un == 1])
    di.close()


def _c5_keys(n, dev, chunk=1 << 27):
    ks, vs = [], []
    for s0 in range(0, n, chunk):
        idx = torch.arange(s0, min(n, s0 + chunk), dtype=torch.int64, device=dev)
        ks.append(W.splitmix64_torch(W.SEED_KEYS + 5, idx).cpu())
        vs.append(W.values_torch(W.SEED_VALUES + 5, s0, idx.shape[0], dev).cpu())
    return torch.cat(ks).numpy().view(np.uint64), torch.cat(vs).numpy().view(np.uint64)


def _c5_updates_on(keyset, rnd, n, R, chunk=1 << 26):
    """(keys, values) of round `rnd`'s update ops whose key is in `keyset` (sorted
    u64), in global op order -- the only ops of the round that can change those keys.
    The ops are drawn with the generator's torch twin on the device (pinned bit for
    bit to the numpy generator, tests/test_workloads.py) and only selected there;
    the replay itself is the CPU oracle's."""
    ks_d = torch.from_numpy(keyset.view(np.int64)).to(DEV)
    ks, vs = [], []
    for s0 in range(rnd * R, (rnd + 1) * R, chunk):
        k, u, v = W.mixed_ops_torch(5, n, s0, chunk, DEV)
        m = (u == 1) & torch.isin(k, ks_d)
        ks.append(k[m].cpu().numpy().view(np.uint64))
        vs.append(v[m].cpu().numpy().view(np.uint64))
    return np.concatenate(ks), np.concatenate(vs)


@pytest.mark.slow
def test_c5_full_size_rounds():
    """Config 5 at its configured size on one GPU, as bench.py --config c5 runs it:
    2^30 random u64 keys, rounds of 2^29 mixed ops (90% lookups at 50% hit, 10%
    updates) through the multi-GPU layer at one rank (reading C7).
    * round 0: EVERY op against its closed form (no update precedes it: a hit
      returns the key's build value vals[pick], a miss CUART_MISS, an update op
      CUART_MISS);
    * round 1: a 10^6-op sample against the plain-map oracle replaying every
      round-0 update on the sampled keys (the only ops that can change them);
    * the state after both rounds: 10^6 sampled keys against the same replay."""
    n, R = W.C5.n_keys, W.C5_ROUND
    keys, vals = _c5_keys(n, DEV)
    from paper_conf_icpp_koppehelggp21_b200.dist import DistIndex
    di = DistIndex(keys, vals, mode="range", transport="p2p", rank=0, world=1)
    outs = []
    for rnd in range(2):
        k, u, v = W.mixed_ops_torch(5, n, rnd * R, R, DEV)
        outs.append(di.mixed_round(k, v, u, fused=rnd == 1))      # round 1 through cuart_dist_mixed
        del k, u, v
    rng = np.random.default_rng(55)
    probe = np.sort(rng.choice(n, 1_000_000, replace=False))
    pk = keys[probe]
    out_p = di.lookup(torch.from_numpy(pk.view(np.int64)).to(DEV))
    torch.cuda.synchronize()
    # round 0, every op, closed form (on the device, chunked)
    vals_d = torch.from_numpy(vals.view(np.int64)).to(DEV)
    for s0 in range(0, R, 1 << 26):
        j = torch.arange(s0, s0 + (1 << 26), dtype=torch.int64, device=DEV)
        upd = W._t_ult(W.splitmix64_torch(W.SEED_UPDATES + 5, 3 * j), int(W.C5_UPDATE_P * 2**64))
        pick = W._t_umod(W.splitmix64_torch(W.SEED_UPDATES + 5, 3 * j + 1), n)
        hit = W._t_ult(W.splitmix64_torch(W.SEED_QUERIES + 5, 2 * j), 1 << 63)
        exp = torch.where(hit & ~upd, vals_d[pick], torch.full_like(j, -1))
        assert torch.equal(outs[0][s0: s0 + (1 << 26)], exp), s0
    del vals_d
    # round 1, sampled, vs the plain-map replay of round 0's updates on the sampled keys
    js = np.sort(rng.choice(R, 1_000_000, replace=False)).astype(np.uint64) + np.uint64(R)
    k1, u1, _ = W.mixed_ops(5, n, js)
    # key index of every op (hits and updates draw key #pick; misses draw absent keys)
    pick1 = (W.splitmix64(W.SEED_UPDATES + 5, np.uint64(3) * js + np.uint64(1)) % np.uint64(n)).astype(np.int64)
    hit1 = W.splitmix64(W.SEED_QUERIES + 5, np.uint64(2) * js) < np.uint64(1 << 63)
    idx = np.concatenate([pick1[(u1 == 0) & hit1], probe])
    assert np.array_equal(keys[pick1[(u1 == 0) & hit1]], k1[(u1 == 0) & hit1])
    sub = MapOracle(keys[idx], vals[idx])                  # build values of the sampled keys
    ks_sorted = np.unique(keys[idx])
    uk0, uv0 = _c5_updates_on(ks_sorted, 0, n, R)
    sub.update(uk0, uv0)
    exp1 = sub.lookup(k1)
    exp1[u1 == 1] = OART_MISS
    got1 = outs[1][torch.from_numpy((js - np.uint64(R)).astype(np.int64)).to(DEV)].cpu().numpy().view(np.uint64)
    assert np.array_equal(got1, exp1)
    assert abs((exp1[u1 == 0] != OART_MISS).mean() - 0.5) < 0.01
    # the state after both rounds on the probe keys
    uk1, uv1 = _c5_updates_on(ks_sorted, 1, n, R)
    sub.update(uk1, uv1)
    assert np.array_equal(out_p.cpu().numpy().view(np.uint64), sub.lookup(pk))
    di.close()
