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
