"""Multi-process (world_size 2, gloo, CPU) tests of the multi-GPU protocol in
paper_conf_icpp_koppehelggp21_b200/dist.py: splitters, routing order, the
count + run all-to-all exchange, reassembly, and global (rank-major) update
order in both replica and range-partitioned modes.  The per-rank local engine
is the CPU oracle and routing is a numpy test double; on the GPU the same
protocol runs with the CuART kernels over NCCL (tests/test_gpu_route.py covers
the kernels)."""
import os
import socket
import tempfile

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle import ArtOracle, MapOracle, OART_MISS


class NumpyOps:
    device = torch.device("cpu")

    def build(self, keys, values, lut_bytes):
        return ArtOracle(keys, values)

    def tensor(self, a):
        return torch.from_numpy(np.ascontiguousarray(a))

    def route(self, keys, lens, values, splitters, nparts):
        from paper_conf_icpp_koppehelggp21_b200.dist import owners, prefix8
        k = keys.numpy()
        if k.dtype == np.int64:
            k = k.view(np.uint64)
        elif k.dtype == np.int32:
            k = k.view(np.uint32)
        pre = prefix8((k, lens.numpy()) if lens is not None else k)
        own = owners(pre, splitters.numpy().view(np.uint64))
        order = np.argsort(own, kind="stable")
        perm = np.empty(order.shape[0], np.int64)
        perm[order] = np.arange(order.shape[0])
        counts = np.bincount(own, minlength=nparts).astype(np.int64)
        sk = torch.from_numpy(keys.numpy()[order].copy())
        sl = torch.from_numpy(lens.numpy()[order].copy()) if lens is not None else None
        sv = torch.from_numpy(values.numpy()[order].copy()) if values is not None else None
        return sk, sl, sv, torch.from_numpy(perm), torch.from_numpy(counts)

    def unroute(self, res, perm):
        return res[perm]

    def _np(self, keys, lens):
        k = keys.numpy()
        if k.dtype == np.int64:
            return k.view(np.uint64)
        if k.dtype == np.int32:
            return k.view(np.uint32)
        if lens is not None:
            return (k, lens.numpy())
        return k

    def lookup(self, index, keys, lens):
        if keys.shape[0] == 0:
            return torch.zeros(0, dtype=torch.int64)
        return torch.from_numpy(index.lookup(self._np(keys, lens)).view(np.int64))

    def update(self, index, keys, lens, values):
        if keys.shape[0]:
            index.update(self._np(keys, lens), values.numpy().view(np.uint64))

    def close(self, index):
        index.close()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, mode, kind, outdir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icpp_koppehelggp21_b200.dist import DistIndex
    keys, vals, q, (uk, uv) = _data(kind, rank, world)
    di = DistIndex(keys, vals, mode=mode, ops=NumpyOps())
    ops = di.ops
    res = di.lookup(_t(q))
    di.update((_t(uk), torch.from_numpy(uv.view(np.int64))))
    res2 = di.lookup(_t(keys))       # every rank looks up the whole key set after the global update
    np.save(os.path.join(outdir, f"r{rank}_res.npy"), res.numpy())
    np.save(os.path.join(outdir, f"r{rank}_res2.npy"), res2.numpy())
    np.save(os.path.join(outdir, f"r{rank}_nlocal.npy"), np.array([di.n_local_keys]))
    di.close()
    dist.destroy_process_group()


def _t(a):
    if isinstance(a, tuple):
        return (torch.from_numpy(a[0]), torch.from_numpy(a[1]))
    if a.dtype == np.uint64:
        return torch.from_numpy(a.view(np.int64))
    if a.dtype == np.uint32:
        return torch.from_numpy(a.view(np.int32))
    return torch.from_numpy(a)


def _data(kind, rank, world):
    import workloads as W
    if kind == "u64":
        cfg = W.CONFIGS["c1"]
        keys, vals = W.build_set(cfg)
        q = W.lookup_batch(cfg, keys, rank * 20_000, 20_000)
        uk, uv = W.update_batch(cfg, keys, rank * 30_000, 30_000)
        return keys, vals, q, (uk, uv)
    if kind == "u32dense":
        n = 1 << 14
        keys = np.arange(n, dtype=np.uint32)
        vals = keys.astype(np.uint64) * 3 + 1
        rng = np.random.default_rng(rank)
        q = rng.integers(0, n + 500, 5000, dtype=np.uint32)
        uk = rng.integers(0, n + 100, 6000, dtype=np.uint32)
        uv = rng.integers(0, 1 << 62, 6000, dtype=np.uint64)
        return keys, vals, q, (uk, uv)
    slots, lens = W.string_keys(4, 5000)
    vals = np.arange(5000, dtype=np.uint64) + 7
    rng = np.random.default_rng(10 + rank)
    qi = rng.integers(0, 5000, 3000)
    q = (slots[qi].copy(), lens[qi].copy())
    ui = rng.integers(0, 5000, 4000)
    uv = rng.integers(0, 1 << 62, 4000, dtype=np.uint64)
    return (slots, lens), vals, q, ((slots[ui].copy(), lens[ui].copy()), uv)


@pytest.mark.parametrize("mode", ["range", "replica"])
@pytest.mark.parametrize("kind", ["u64", "u32dense", "bytes"])
def test_dist_protocol_world2(mode, kind):
    world = 2
    with tempfile.TemporaryDirectory() as d:
        mp.start_processes(_worker, args=(world, _free_port(), mode, kind, d), nprocs=world, start_method="spawn")
        # reference: one map over the global key set; lookups per rank shard, then all
        # ranks' update batches applied in rank-major global order (reading C7)
        keys, vals, _, _ = _data(kind, 0, world)
        ref = MapOracle(keys, vals)
        for r in range(world):
            _, _, q, _ = _data(kind, r, world)
            got = np.load(os.path.join(d, f"r{r}_res.npy")).view(np.uint64)
            assert np.array_equal(got, ref.lookup(q)), (mode, kind, r)
        for r in range(world):
            _, _, _, (uk, uv) = _data(kind, r, world)
            ref.update(uk, uv)
        exp = ref.lookup(keys)
        for r in range(world):
            assert np.array_equal(np.load(os.path.join(d, f"r{r}_res2.npy")).view(np.uint64), exp)
        nloc = [int(np.load(os.path.join(d, f"r{r}_nlocal.npy"))[0]) for r in range(world)]
        n = keys[0].shape[0] if isinstance(keys, tuple) else keys.shape[0]
        if mode == "range":
            assert sum(nloc) == n
            assert min(nloc) > 0.4 * n / world        # quantile splitters balance (incl. dense u32)
        else:
            assert nloc == [n] * world


def test_splitters_skip_common_prefix():
    from paper_conf_icpp_koppehelggp21_b200.dist import compute_splitters, owners, prefix8
    keys = np.arange(1 << 16, dtype=np.uint32)              # all share leading bytes 00 00
    pre = prefix8(keys)
    for p in (2, 4, 8):
        sp = compute_splitters(pre, p)
        cnt = np.bincount(owners(pre, sp), minlength=p)
        assert cnt.min() == cnt.max() == (1 << 16) // p
    # equal 8-byte prefixes never straddle partitions
    slots = np.zeros((10, 32), np.uint8)
    slots[:, :8] = 7
    slots[:, 8] = np.arange(10)
    lens = np.full(10, 9, np.uint8)
    own = owners(prefix8((slots, lens)), compute_splitters(prefix8((slots, lens)), 4))
    assert len(set(own.tolist())) == 1


# ------------------------------------------------------------------ mixed rounds (config 5, reading C7)
def _np_partition(self, keys, lens, values, flags):
    f = flags.numpy().astype(bool)
    order = np.argsort(f, kind="stable")
    perm = np.empty(order.shape[0], np.int64)
    perm[order] = np.arange(order.shape[0])
    counts = np.array([(~f).sum(), f.sum()], np.int64)
    return (torch.from_numpy(keys.numpy()[order].copy()),
            torch.from_numpy(lens.numpy()[order].copy()) if lens is not None else None,
            torch.from_numpy(values.numpy()[order].copy()), torch.from_numpy(perm), torch.from_numpy(counts))


NumpyOps.partition = _np_partition
MIX_KEYS, MIX_ROUND, MIX_ROUNDS = 1 << 14, 1 << 13, 3


def _mixed_worker(rank, world, port, mode, outdir):
    import workloads as W
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_icpp_koppehelggp21_b200.dist import DistIndex
    keys = W.u64_keys(5, MIX_KEYS)
    vals = W.values_for(W.SEED_VALUES + 5, np.arange(MIX_KEYS, dtype=np.uint64))
    di = DistIndex(keys, vals, mode=mode, ops=NumpyOps())
    per = MIX_ROUND // world
    outs = []
    for r in range(MIX_ROUNDS):
        start = r * MIX_ROUND + rank * per
        k, u, v = W.mixed_ops(5, MIX_KEYS, np.arange(start, start + per))
        out = di.mixed_round(torch.from_numpy(k.view(np.int64)), torch.from_numpy(v.view(np.int64)),
                             torch.from_numpy(u))
        outs.append(out.numpy())
    np.save(os.path.join(outdir, f"mix_r{rank}.npy"), np.concatenate(outs))
    di.close()
    dist.destroy_process_group()


def _replay(world):
    """Oracle replay of reading C7: per round, all lookups see the pre-round state,
    then the round's updates apply in global op order."""
    import workloads as W
    keys = W.u64_keys(5, MIX_KEYS)
    o = MapOracle(keys, W.values_for(W.SEED_VALUES + 5, np.arange(MIX_KEYS, dtype=np.uint64)))
    per = MIX_ROUND // world
    res = {r: [] for r in range(world)}
    for rnd in range(MIX_ROUNDS):
        k, u, v = W.mixed_ops(5, MIX_KEYS, np.arange(rnd * MIX_ROUND, (rnd + 1) * MIX_ROUND))
        look = o.lookup(k)
        look[u == 1] = OART_MISS
        for r in range(world):
            res[r].append(look[r * per:(r + 1) * per])
        o.update(k[u == 1], v[u == 1])
    return {r: np.concatenate(x) for r, x in res.items()}


@pytest.mark.parametrize("mode", ["range", "replica"])
def test_mixed_rounds_world2_p_independent(mode):
    world = 2
    with tempfile.TemporaryDirectory() as d:
        mp.start_processes(_mixed_worker, args=(world, _free_port(), mode, d), nprocs=world, start_method="spawn")
        exp = _replay(world)
        for r in range(world):
            assert np.array_equal(np.load(os.path.join(d, f"mix_r{r}.npy")).view(np.uint64), exp[r])
        # P-independence: the concatenation equals the single-rank replay
        one = _replay(1)[0]
        both = np.concatenate([np.load(os.path.join(d, f"mix_r{r}.npy")).view(np.uint64).reshape(MIX_ROUNDS, -1)
                               for r in range(world)], axis=1).ravel()
        assert np.array_equal(both, one)
