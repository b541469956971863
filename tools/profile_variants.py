"""Run one k_lookup per LUT format on config c3 (for ncu -k regex:k_lookup)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_koppehelggp21_b200 as C  # noqa: E402
import workloads as W  # noqa: E402

cfg = W.CONFIGS[os.environ.get("CFG", "c3")]
dev = torch.device("cuda:0")
keys_d = W.u64_keys_torch(W.config_id(cfg), cfg.n_keys, dev)
keys = keys_d.cpu().numpy().view(np.uint64)
vals = W.values_for(W.SEED_VALUES + W.config_id(cfg), np.arange(cfg.n_keys, dtype=np.uint64))
lay = C.Layout(keys, vals, lut_bytes=3)
m = 1 << 28
q = W.lookup_batch_torch(cfg, keys_d, 0, m, device=dev)
out = torch.empty(m, dtype=torch.int64, device=dev)
for fmt in [int(x) for x in os.environ.get("FORMATS", "1,2,3").split(",")]:
    ix = C.Index.from_layout(lay, device=0, lut_format=fmt)
    ix.lookup(q, out)
    torch.cuda.synchronize()
    print("format", fmt, "done", flush=True)
    ix.close()
