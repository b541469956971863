"""World-size-2 tests (gloo, CPU) of the multi-GPU layer's host side.

* cuart_dist_partition through the library's host bootstrap: both processes hand
  the C library a torch.distributed all-gather (dist.TorchAllGather), the library
  all-gathers its splitters and checks that every rank agrees; ownership is
  complete, disjoint and balanced (quantile splitters, dense u32 keys included); a
  rank with different splitters makes the collective fail on every rank.
* The exchange arithmetic of cuart_dist_update / cuart_dist_lookup, emulated with
  numpy per rank and real collectives between the processes: chunked batches, the
  per-chunk count matrix, cuart_dist_chunk_plan's offsets, priorities
  rank * 2^32 / P + op index, one update epoch per call with a winner check per
  chunk (csrc/dist.cu).  The result must equal the plain-map oracle applying the
  concatenated batches in rank-major order (reading C7), for range and replica
  modes, with ragged and empty batches and dropped reserved-value ops.
The device kernels of the same path are covered by tests/test_gpu_dist.py."""
import os
import socket
import tempfile

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle import MapOracle, OART_MISS


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _init(rank, world, port):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)


def _keyset(kind):
    import workloads as W
    if kind == "u64":
        return W.u64_keys(1, 1 << 15)
    if kind == "u32dense":
        return np.arange(1 << 14, dtype=np.uint32)               # all share the leading bytes 00 00
    return W.string_keys(4, 6000)


# ------------------------------------------------------------------ partition + bootstrap
def _partition_worker(rank, world, port, kind, outdir, bad):
    _init(rank, world, port)
    from paper_conf_icpp_koppehelggp21_b200 import _binding as B
    from paper_conf_icpp_koppehelggp21_b200.dist import TorchAllGather, partition
    keys = _keyset(kind)
    sp = None
    if bad:
        sp = np.array([1 << 62 if rank == 0 else 1 << 61], np.uint64)
    try:
        s, own = partition(keys, rank, world, splitters=sp, gather=TorchAllGather())
        np.save(os.path.join(outdir, f"sp{rank}.npy"), s)
        np.save(os.path.join(outdir, f"own{rank}.npy"), own)
    except B.CuartError as e:
        np.save(os.path.join(outdir, f"err{rank}.npy"), np.array([e.status]))
    dist.destroy_process_group()


@pytest.mark.parametrize("kind", ["u64", "u32dense", "bytes"])
def test_partition_world2(kind):
    world = 2
    with tempfile.TemporaryDirectory() as d:
        mp.start_processes(_partition_worker, args=(world, _free_port(), kind, d, False), nprocs=world,
                           start_method="spawn")
        sps = [np.load(os.path.join(d, f"sp{r}.npy")) for r in range(world)]
        owns = [np.load(os.path.join(d, f"own{r}.npy")) for r in range(world)]
        assert np.array_equal(sps[0], sps[1]) and np.array_equal(owns[0], owns[1])
        from paper_conf_icpp_koppehelggp21_b200.dist import owners, prefix8
        keys = _keyset(kind)
        assert np.array_equal(owns[0], owners(prefix8(keys), sps[0]))
        cnt = np.bincount(owns[0], minlength=world)
        n = owns[0].shape[0]
        assert cnt.sum() == n and cnt.min() > 0.45 * n          # quantile splitters balance


def test_partition_disagreement_fails_everywhere():
    world = 2
    with tempfile.TemporaryDirectory() as d:
        mp.start_processes(_partition_worker, args=(world, _free_port(), "u64", d, True), nprocs=world,
                           start_method="spawn")
        for r in range(world):
            assert int(np.load(os.path.join(d, f"err{r}.npy"))[0]) == 1    # CUART_ERR_INVALID_ARGUMENT


# ------------------------------------------------------------------ emulated exchange
CHUNK = 700


def _exchange(payload):
    out = [None] * dist.get_world_size()
    dist.all_gather_object(out, payload)
    return out


def _emulated_update(state, keys, vals, splitters, mode):
    """One cuart_dist_update call as csrc/dist.cu runs it, with numpy standing in for
    the kernels: state = (sorted keys of this rank's index, values, winner words)."""
    from paper_conf_icpp_koppehelggp21_b200.dist import chunk_plan, owners, prefix8
    P, me = dist.get_world_size(), dist.get_rank()
    n = keys.shape[0]
    nmax = max(_exchange(n))                                    # the per-call n round
    nc = (nmax + CHUNK - 1) // CHUNK
    ikeys, ivals, win = state
    epoch = win["epoch"] = win["epoch"] + 1                     # one epoch for the whole call
    for c in range(nc):
        b0 = c * CHUNK
        k, v = keys[b0:b0 + CHUNK], vals[b0:b0 + CHUNK]
        prio = me * ((1 << 32) // P) + b0 + np.arange(k.shape[0], dtype=np.int64)
        own = np.zeros(k.shape[0], np.int64) if mode == "replica" else owners(prefix8(k), splitters)
        order = np.argsort(own, kind="stable")                  # send order
        row = [k.shape[0]] * P if mode == "replica" else np.bincount(own, minlength=P).tolist()
        M = np.array(_exchange(row), np.uint64)                 # k_publish / k_wait_counts
        seg, _, push = chunk_plan(M, me)
        sent = [(k[order], v[order], prio[order], own[order])]
        allsent = _exchange(sent[0])                            # the fused push
        # owner: the receive window = sources' runs in rank order
        rk, rv, rp = [], [], []
        for s in range(P):
            sk, sv, spr, so = allsent[s]
            m = np.ones(sk.shape[0], bool) if mode == "replica" else so == me
            rk.append(sk[m]), rv.append(sv[m]), rp.append(spr[m])
        rk, rv, rp = np.concatenate(rk), np.concatenate(rv), np.concatenate(rp)
        assert rk.shape[0] == int(seg[P])
        # stage 1: locate + atomicMax(epoch << 32 | prio); stage 2: the winner writes
        pos = np.searchsorted(ikeys, rk)
        pos_c = np.minimum(pos, ikeys.shape[0] - 1)
        hit = (pos < ikeys.shape[0]) & (ikeys[pos_c] == rk) & (rv != OART_MISS)
        for p_, pr in zip(pos_c[hit], rp[hit]):
            word = (epoch << 32) | int(pr)
            win["w"][p_] = max(win["w"][p_], word)
        for p_, pr, val in zip(pos_c[hit], rp[hit], rv[hit]):
            if win["w"][p_] == ((epoch << 32) | int(pr)):
                ivals[p_] = val


def _emu_worker(rank, world, port, mode, outdir):
    _init(rank, world, port)
    import workloads as W
    from paper_conf_icpp_koppehelggp21_b200.dist import owners, prefix8, partition
    keys = W.u64_keys(5, 1 << 13)
    vals = W.values_for(W.SEED_VALUES + 5, np.arange(keys.shape[0], dtype=np.uint64))
    sp, own = partition(keys, rank, world)
    mine = own == rank if mode == "range" else np.ones(keys.shape[0], bool)
    order = np.argsort(keys[mine])
    state = (keys[mine][order], vals[mine][order].copy(), {"epoch": 0, "w": np.zeros(int(mine.sum()), object)})
    rng = np.random.default_rng(100 + rank)
    outs = []
    for call in range(3):
        m = [1500, 0, 2300][(call + rank) % 3]                 # ragged batches, an empty rank
        pick = rng.integers(0, keys.shape[0], m)
        uk = np.where(rng.random(m) < 0.9, keys[pick], rng.integers(0, 2**63, m, dtype=np.uint64))
        uv = rng.integers(0, 2**62, m, dtype=np.uint64)
        uv[::211] = OART_MISS                                   # reading C5: dropped ops
        _emulated_update(state, uk, uv, sp, mode)
        np.save(os.path.join(outdir, f"ops{rank}_{call}.npy"), np.stack([uk, uv]))
        # lookups of the whole key set after the call, served by the owners
        q = keys
        if mode == "range":
            qo = owners(prefix8(q), sp)
            ans = np.full(q.shape[0], OART_MISS, np.uint64)
            local = qo == rank
            pos = np.searchsorted(state[0], q[local])
            ans[local] = state[1][np.minimum(pos, state[0].shape[0] - 1)]
            allans = _exchange(ans)
            got = np.where(qo == 0, allans[0], allans[1])
        else:
            pos = np.searchsorted(state[0], q)
            got = state[1][pos]
        outs.append(got)
    np.save(os.path.join(outdir, f"res{rank}.npy"), np.stack(outs))
    dist.destroy_process_group()


@pytest.mark.parametrize("mode", ["range", "replica"])
def test_emulated_exchange_world2_rank_major(mode):
    import workloads as W
    world = 2
    with tempfile.TemporaryDirectory() as d:
        mp.start_processes(_emu_worker, args=(world, _free_port(), mode, d), nprocs=world, start_method="spawn")
        keys = W.u64_keys(5, 1 << 13)
        o = MapOracle(keys, W.values_for(W.SEED_VALUES + 5, np.arange(keys.shape[0], dtype=np.uint64)))
        for call in range(3):
            for r in range(world):                              # rank-major global order (reading C7)
                uk, uv = np.load(os.path.join(d, f"ops{r}_{call}.npy"))
                o.update(uk, uv)
            exp = o.lookup(keys)
            for r in range(world):
                assert np.array_equal(np.load(os.path.join(d, f"res{r}.npy"))[call], exp), (mode, call, r)
