"""The complete multi-GPU path (cuart_dist_build / _lookup / _update, transport
P2P) as 2 processes sharing cuda:0: the library's host bootstrap runs over
torch.distributed (gloo) through the callback in cfg; each process maps the
other's receive windows and control block with CUDA IPC (same device here,
NVLink peers on a multi-GPU box); the fused scatter stores ops into the owner's
window, the owner's walk stores results into the requester's window, and the
ranks order each other with device-side flags.  (NCCL refuses two ranks on one
device, so transport NCCL runs at one rank, tests/test_gpu_dist.py.)  Range and
replica modes, lookups, updates and mixed rounds; results equal the single-index
oracle."""
import os
import socket
import tempfile

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle import MapOracle, OART_MISS

pytestmark = pytest.mark.gpu
N_KEYS, N_Q, N_U, ROUND = 1 << 18, 1 << 20, 1 << 18, 1 << 20


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, mode, outdir):
    import workloads as W
    from paper_conf_icpp_koppehelggp21_b200.dist import DistIndex
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    dev = torch.device("cuda:0")
    cfg = W.Config("cX", "u64", N_KEYS, N_Q, N_U, 0.5, "")
    keys = W.u64_keys(3, N_KEYS)
    vals = W.values_for(W.SEED_VALUES + 3, np.arange(N_KEYS, dtype=np.uint64))
    torch.cuda.set_device(dev)
    di = DistIndex(keys, vals, mode=mode, transport="p2p", chunk=1 << 18)
    kd = torch.from_numpy(keys.view(np.int64)).to(dev)
    q = W.lookup_batch_torch(W.CONFIGS["c3"], kd, rank * N_Q, N_Q, device=dev)
    r1 = di.lookup(q)
    uk, uv = W.update_batch_torch(W.CONFIGS["c3"], kd, rank * N_U, N_U)
    di.update(uk, uv)
    r2 = di.lookup(kd)
    per = ROUND // world
    k, u, v = W.mixed_ops_torch(5, N_KEYS, rank * per, per, dev)
    # mixed round over the c3 key set: keys drawn by index from c5's stream, remapped to this set
    k = torch.where(u.bool(), kd[W._t_umod(k, N_KEYS)], k)
    r3 = di.mixed_round(k, v, u)
    torch.cuda.synchronize()
    for name, t in (("r1", r1), ("r2", r2), ("r3", r3), ("k3", k), ("u3", u), ("v3", v)):
        np.save(os.path.join(outdir, f"{name}_{rank}.npy"), t.cpu().numpy())
    di.close()
    dist.destroy_process_group()


@pytest.mark.parametrize("mode", ["range", "replica"])
def test_two_processes_one_gpu(mode):
    import workloads as W
    world = 2
    with tempfile.TemporaryDirectory() as d:
        mp.start_processes(_worker, args=(world, _port(), mode, d), nprocs=world, start_method="spawn")
        keys = W.u64_keys(3, N_KEYS)
        vals = W.values_for(W.SEED_VALUES + 3, np.arange(N_KEYS, dtype=np.uint64))
        o = MapOracle(keys, vals)
        for r in range(world):
            q = W.lookup_batch(W.CONFIGS["c3"], keys, r * N_Q, N_Q)
            assert np.array_equal(np.load(os.path.join(d, f"r1_{r}.npy")).view(np.uint64), o.lookup(q))
        for r in range(world):                                  # global rank-major update order
            uk, uv = W.update_batch(W.CONFIGS["c3"], keys, r * N_U, N_U)
            o.update(uk, uv)
        exp = o.lookup(keys)
        for r in range(world):
            assert np.array_equal(np.load(os.path.join(d, f"r2_{r}.npy")).view(np.uint64), exp)
        ks = [np.load(os.path.join(d, f"k3_{r}.npy")).view(np.uint64) for r in range(world)]
        us = [np.load(os.path.join(d, f"u3_{r}.npy")) for r in range(world)]
        vs = [np.load(os.path.join(d, f"v3_{r}.npy")).view(np.uint64) for r in range(world)]
        for r in range(world):                                  # lookups see the pre-round state
            e = o.lookup(ks[r])
            e[us[r] == 1] = OART_MISS
            assert np.array_equal(np.load(os.path.join(d, f"r3_{r}.npy")).view(np.uint64), e)
