"""Debug driver: one cuart_dist index at world size 1 (main thread), lookups + an update."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import workloads as W  # noqa: E402
from paper_conf_icpp_koppehelggp21_b200.dist import DistIndex  # noqa: E402
from oracle import MapOracle  # noqa: E402

transport = sys.argv[1] if len(sys.argv) > 1 else "p2p"
n = 40_000
keys = W.u64_keys(7, n)
vals = W.values_for(W.SEED_VALUES + 7, np.arange(n, dtype=np.uint64))
print("build", flush=True)
di = DistIndex(keys, vals, mode="range", transport=transport, rank=0, world=1, chunk=8192)
print("built", flush=True)
kd = torch.from_numpy(keys.view(np.int64)).cuda()
out = di.lookup(kd)
torch.cuda.synchronize()
print("lookup ok", np.array_equal(out.cpu().numpy().view(np.uint64), vals), di.last(), flush=True)
uv = torch.arange(n, dtype=torch.int64, device="cuda") + 5
di.update(kd, uv)
out = di.lookup(kd)
torch.cuda.synchronize()
print("update ok", np.array_equal(out.cpu().numpy(), uv.cpu().numpy()), flush=True)
di.close()
print("closed", flush=True)
