"""The seeded generators: numpy and torch twins agree bit for bit; recipe properties."""
import numpy as np
import torch

import workloads as W


def test_splitmix64_reference_values():
    # splitmix64 stream with state starting at 0: first outputs (Vigna's reference generator)
    assert W.splitmix64_scalar(0, 0) == 0xE220A8397B1DCDAF
    assert W.splitmix64_scalar(0, 1) == 0x6E789E6AA1B965F4
    assert int(W.splitmix64(0, np.array([0, 1], np.uint64))[1]) == 0x6E789E6AA1B965F4


def test_torch_twin_matches_numpy():
    c = W.CONFIGS["c1"]
    keys, _ = W.build_set(c)
    tk = W.u64_keys_torch(1, c.n_keys, "cpu")
    assert np.array_equal(tk.numpy().view(np.uint64), keys)
    q = W.lookup_batch(c, keys, 1000, 5000)
    tq = W.lookup_batch_torch(c, torch.from_numpy(keys.view(np.int64)), 1000, 5000)
    assert np.array_equal(tq.numpy().view(np.uint64), q)
    uk, uv = W.update_batch(c, keys, 7, 3000)
    tuk, tuv = W.update_batch_torch(c, torch.from_numpy(keys.view(np.int64)), 7, 3000)
    assert np.array_equal(tuk.numpy().view(np.uint64), uk)
    assert np.array_equal(tuv.numpy().view(np.uint64), uv)
    c2 = W.CONFIGS["c2"]
    q2 = W.lookup_batch(c2, None, 0, 4096)
    tq2 = W.lookup_batch_torch(c2, torch.zeros(1, dtype=torch.int64), 0, 4096)
    assert np.array_equal(tq2.numpy().view(np.uint32), q2)


def test_recipe_properties():
    c = W.CONFIGS["c1"]
    keys, vals = W.build_set(c)
    assert np.unique(keys).shape[0] == keys.shape[0]            # bijective counter draw
    assert not np.any(vals == W.RESERVED_VALUE)
    absent = W.u64_absent_keys(1, c.n_keys, 0, 100_000)
    assert np.intersect1d(absent, keys).shape[0] == 0
    q = W.lookup_batch(c, keys, 0, 100_000)
    frac = np.isin(q, keys).mean()
    assert abs(frac - 0.5) < 0.01
    uk, uv = W.update_batch(c, keys)
    assert abs(np.isin(uk, keys).mean() - 0.9) < 0.01


def test_string_keys_prefix_free_and_distinct():
    slots, lens = W.string_keys(4, 20_000)
    assert slots.shape == (20_000, 32)
    assert lens.min() >= 8 and lens.max() <= 32
    rows = {bytes(slots[i, : lens[i]]) for i in range(len(lens))}
    assert len(rows) == 20_000
    for i in range(0, 20_000, 97):
        k = bytes(slots[i, : lens[i]])
        assert k[-1] == 0 and 0 not in k[:-1]
        assert not slots[i, lens[i]:].any()


def test_string_lookup_torch_twin():
    cfg = W.CONFIGS["c4"]
    slots, lens = W.string_keys(4, 50_000)
    idx = W.string_lookup_at(cfg, 50_000, np.arange(1000, 6000))
    qs, ql = W.string_lookup_torch(cfg, torch.from_numpy(slots), torch.from_numpy(lens), 1000, 5000)
    assert np.array_equal(qs.numpy(), slots[idx]) and np.array_equal(ql.numpy(), lens[idx])
    # Zipf(0.99) skew: the hottest key takes a large share
    assert np.bincount(idx).max() > 100


def test_mixed_ops_twin_and_mix():
    k, u, v = W.mixed_ops(5, 1 << 16, np.arange(100, 50_100))
    tk, tu, tv = W.mixed_ops_torch(5, 1 << 16, 100, 50_000, "cpu")
    assert np.array_equal(tk.numpy().view(np.uint64), k)
    assert np.array_equal(tu.numpy(), u) and np.array_equal(tv.numpy().view(np.uint64), v)
    assert abs(u.mean() - 0.1) < 0.01
    keys = W.u64_keys(5, 1 << 16)
    present = np.isin(k, keys)
    assert present[u == 1].all()                                   # updates target the set
    assert abs(present[u == 0].mean() - 0.5) < 0.02                # lookups: 50% hit


def test_torch_helper_twins():
    """The torch helpers the full-size tests use agree with the numpy generator."""
    cfg = W.CONFIGS["c4"]
    n = 30_000
    idx = W.string_lookup_index_torch(cfg, n, 500, 4000, "cpu", W.zipf_cdf_torch(n, "cpu"),
                                      W.rank_permutation_torch(cfg, n, "cpu"))
    assert np.array_equal(idx.numpy(), W.string_lookup_at(cfg, n, np.arange(500, 4500)))
    v = W.values_torch(W.SEED_VALUES + 5, 123, 5000, "cpu")
    assert np.array_equal(v.numpy().view(np.uint64), W.values_for(W.SEED_VALUES + 5, np.arange(123, 5123, dtype=np.uint64)))
