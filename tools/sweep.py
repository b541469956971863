"""Variant sweep for the lookup/update kernels on one config (device-timed).

    python tools/sweep.py [--config c3] [--reps 5]

For each (LUT entry width, cache policy) it uploads the same host layout and
times cuart_lookup over the full lookup batch and cuart_update over the update
batch with CUDA events.  Results are printed as JSON lines; the chosen defaults
are documented in DESIGN.md with these numbers.
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_icpp_koppehelggp21_b200 as C  # noqa: E402
import workloads as W  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c3")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--lut", type=int, default=3)
    ap.add_argument("--policies", default="0,1,2,3")
    ap.add_argument("--formats", default="1,2,3")
    a = ap.parse_args()
    cfg = W.CONFIGS[a.config]
    dev = torch.device("cuda:0")
    if cfg.kind == "u64":
        keys_d = W.u64_keys_torch(W.config_id(cfg), cfg.n_keys, dev)
        keys = keys_d.cpu().numpy().view(np.uint64)
    else:
        keys = np.arange(cfg.n_keys, dtype=np.uint32)
        keys_d = torch.from_numpy(keys.view(np.int32)).to(dev)
    vals = W.values_for(W.SEED_VALUES + W.config_id(cfg), np.arange(cfg.n_keys, dtype=np.uint64))
    lay = C.Layout(keys, vals, lut_bytes=a.lut)
    q = W.lookup_batch_torch(cfg, keys_d, 0, cfg.n_lookups, device=dev)
    out = torch.empty(cfg.n_lookups, dtype=torch.int64, device=dev)
    ref = None
    if cfg.n_updates:
        uk, uv = W.update_batch_torch(cfg, keys_d)
    for width in [int(x) for x in a.formats.split(",")]:
        for pol in [int(x) for x in a.policies.split(",")]:
            os.environ["CUART_POLICY"] = str(pol)
            ix = C.Index.from_layout(lay, device=0, lut_format=width)
            ix.lookup(q, out)
            torch.cuda.synchronize()
            chk = int(out[: 1 << 24].sum().item())
            if ref is None:
                ref = chk
            ts, tu = [], []
            for _ in range(a.reps):
                e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
                e[0].record()
                ix.lookup(q, out)
                e[1].record()
                if cfg.n_updates:
                    ix.update(uk, uv)
                e[2].record()
                torch.cuda.synchronize()
                ts.append(e[0].elapsed_time(e[1]))
                tu.append(e[1].elapsed_time(e[2]))
            lm = float(np.median(ts))
            um = float(np.median(tu))
            print(json.dumps({"config": a.config, "lut": a.lut, "lut_format": width, "policy": pol,
                              "lookup_ms": round(lm, 3), "mlookups_s": round(cfg.n_lookups / lm / 1e3, 1),
                              "lut_exceptions": ix.stats()["lut_exceptions"], "update_ms": round(um, 3),
                              "mupdates_s": round(cfg.n_updates / um / 1e3, 1) if cfg.n_updates else None,
                              "checksum_ok": chk == ref}), flush=True)
            ix.close()


if __name__ == "__main__":
    main()
