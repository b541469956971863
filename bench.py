#!/usr/bin/env python
"""Benchmark of the CuART hot path on B200 (device-timed), one JSON line on rank 0.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c3] [--impl cuart|reference]

A "step" = one pass of the whole hot path over one batch of the workload:
cuart_lookup over the lookup batch, then cuart_update over the update batch
(the build rows a2-a3 are host-side setup, untimed).
Default workload: BASELINE config 3 (2^26 random u64 keys, 2^30 lookups at 50%
hit + a 2^26-op update batch) — the config that carries both halves of the
metric ("Mlookups/s and Mupdates/s") at 1 and 8 GPUs and fits one B200.

Inputs are resident in HBM before the timed region and are far larger than the
126 MB L2 (8 GiB of queries), so no explicit L2 flush is needed between steps.

N > 1 (torchrun, one process per GPU, NCCL): replica mode — every rank holds the
full index, looks up its own 2^30-query shard of the global stream (weak scaling)
and applies the all-gathered update batches of all ranks in rank-major global
order, so the replicas stay identical.

--impl reference times the CPU oracle (oracle/, single-threaded pointer ART) on
a bounded sample of the same workload: the reference arm for this tier.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402

METRIC = "Mlookups/s and Mupdates/s (device-timed)"
# K-GATHER calibration (tools/kgather*.cu, profiles/r01/): independent random 8-B loads over
# 8 GiB saturate at ~47.5-48 G requests/s on this B200 (each fills a 128-B L2 line from
# DRAM by default), whatever the load flavour; L2-resident (<= 32 MiB) random loads ~245 G/s.
RANDOM_CEILING = {"random_requests_per_s": 47.5e9, "l2_resident_requests_per_s": 245e9,
                  "source": "profiles/r01/kgather*.json"}


def _args():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=10)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--config", default="c3", choices=["c1", "c2", "c3", "c4", "c5"])
    p.add_argument("--impl", default="cuart", choices=["cuart", "reference"])
    p.add_argument("--lut", type=int, default=3)
    p.add_argument("--skip-log2", type=int, default=0,
                   help="byte-string skip table cap (cuart_build_opts.skip_log2; 0 = library choice)")
    p.add_argument("--lut-format", default="auto", choices=["auto", "links", "compact32", "rank"],
                   help="device form of the root table (cuart_build_opts.lut_format)")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--e2e-steps", type=int, default=2)
    p.add_argument("--mode", default="range", choices=["range", "replica"], help="multi-GPU mode (N > 1)")
    p.add_argument("--transport", default="p2p", choices=["p2p", "nccl"],
                   help="range mode exchange: p2p = fused push/return over peer memory (CUDA IPC, NVLink), "
                        "nccl = route + all-to-all")
    p.add_argument("--dist", action="store_true",
                   help="N = 1 through the multi-GPU layer (cuart_dist_*, one rank): its protocol overhead")
    p.add_argument("--l2-persist", type=int, default=0,
                   help="cuart_build_opts.l2_persist: persisting L2 window over the root tables")
    p.add_argument("--c5-fused", type=int, default=0,
                   help="c5 rounds through cuart_dist_mixed (1) or partition + lookup + update + unroute (0)")
    p.add_argument("--c5-share", type=int, default=0,
                   help="c5 on one GPU: the per-GPU share of a P-GPU run (rank 0's keys and owned ops)")
    p.add_argument("--traffic", type=float, default=None,
                   help="ncu dram__bytes_read+write per k_lookup launch (GB), from profiles/, echoed into roofline")
    return p.parse_args()


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi sampling of SM clocks + throttle reasons during the timed region."""
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, dev_index: int):
        self.dev = dev_index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                                          "-i", str(self.dev), "-lms", "100"], stdout=subprocess.PIPE,
                                         stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [x.strip() for x in ln.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------ oracle timing (CPU)
def oracle_timing(cfg, keys, vals, n_lookup_sample, n_update_sample, allcore_factor=8):
    """The oracle as it stands (SURVEY §8(d) CPU-baseline plan), on this box's host cores:
    single-threaded lookups and sequential updates pinned to one core, then the
    read-only lookups fanned over every core (oart_lookup_batch_mt).  Returns
    (mixed 1-core Mops/s, detail)."""
    from oracle import ArtOracle
    t0 = time.perf_counter()
    if isinstance(keys, tuple):
        o = ArtOracle(keys, vals)
    else:   # insertion order does not change the tree (pinned); sorted inserts build faster
        order = np.argsort(keys)
        o = ArtOracle(keys[order], vals[order])
    build_s = time.perf_counter() - t0
    q = host_lookups(cfg, keys, 0, n_lookup_sample)
    uk, uv = W.update_batch(cfg, keys, 0, n_update_sample) if cfg.n_updates and n_update_sample else (None, None)
    cores = sorted(os.sched_getaffinity(0))
    os.sched_setaffinity(0, {cores[0]})             # one core (taskset)
    try:
        t0 = time.perf_counter()
        o.lookup(q)
        t_look = time.perf_counter() - t0
        t_upd = 0.0
        if uk is not None:
            t0 = time.perf_counter()
            o.update(uk, uv)
            t_upd = time.perf_counter() - t0
    finally:
        os.sched_setaffinity(0, set(cores))
    qa = host_lookups(cfg, keys, n_lookup_sample, n_lookup_sample * allcore_factor)
    t0 = time.perf_counter()
    o.lookup_mt(qa, len(cores))
    t_all = time.perf_counter() - t0
    o.close()
    nu = n_update_sample if uk is not None else 0
    mixed = (n_lookup_sample + nu) / (t_look + t_upd) / 1e6
    return mixed, {"build_s": round(build_s, 2), "sample_lookups": n_lookup_sample, "sample_updates": nu,
                   "seconds": round(t_look + t_upd, 3),
                   "oracle_lookup_mops_1core": round(n_lookup_sample / t_look / 1e6, 3),
                   "oracle_update_mops_1core": round(nu / t_upd / 1e6, 3) if nu else None,
                   "oracle_lookup_mops_allcores": round(qa_len(qa) / t_all / 1e6, 3),
                   "allcore_sample_lookups": qa_len(qa), "host_cores": len(cores)}


def layout_engine_timing(cfg, keys, layout, n1, det, allcore_factor=8):
    """§8 f3 (§4.2, Fig. 7): the paper's CPU lookup engine over the flat CuART
    layout (cuart_layout_lookup, product code; OpenMP) on the same query samples as
    the oracle's 1-core and all-core lookups, so the two CPU rates compare the flat
    type-segregated layout against the pointer ART on this host."""
    cores = sorted(os.sched_getaffinity(0))
    q1 = host_lookups(cfg, keys, 0, n1)
    os.sched_setaffinity(0, {cores[0]})
    try:
        t0 = time.perf_counter()
        layout.lookup(q1, threads=1)
        t1 = time.perf_counter() - t0
    finally:
        os.sched_setaffinity(0, set(cores))
    qa = host_lookups(cfg, keys, n1, n1 * allcore_factor)
    t0 = time.perf_counter()
    layout.lookup(qa, threads=len(cores))
    ta = time.perf_counter() - t0
    r1, ra = n1 / t1 / 1e6, qa_len(qa) / ta / 1e6
    return {"kind": "cuart_layout_lookup (flat layout, CPU)", "lookup_mops_1core": round(r1, 3),
            "lookup_mops_allcores": round(ra, 3), "threads": len(cores),
            "vs_oracle_1core": round(r1 / det["oracle_lookup_mops_1core"], 3),
            "vs_oracle_allcores": round(ra / det["oracle_lookup_mops_allcores"], 3)}


def qa_len(q):
    return q[1].shape[0] if isinstance(q, tuple) else q.shape[0]


def host_lookups(cfg, keys, start, m):
    if isinstance(keys, tuple):
        idx = W.string_lookup_at(cfg, keys[1].shape[0], np.arange(start, start + m))
        return (keys[0][idx], keys[1][idx])
    return W.lookup_batch(cfg, keys, start, m)


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    cfg = W.CONFIGS[args.config]
    keys, vals = W.build_set(cfg)
    from oracle import ArtOracle
    t0 = time.perf_counter()
    if isinstance(keys, tuple):
        o = ArtOracle(keys, vals)
    else:   # insertion order does not change the tree (pinned); sorted inserts build faster
        order = np.argsort(keys)
        o = ArtOracle(keys[order], vals[order])
    build_s = time.perf_counter() - t0
    # bounded sample per step, same lookup:update mix as the workload
    nl = min(cfg.n_lookups, 1 << 20)
    nu = min(cfg.n_updates, max(1, nl * cfg.n_updates // cfg.n_lookups)) if cfg.n_updates else 0
    times = []
    for s in range(args.warmup + args.steps):
        q = host_lookups(cfg, keys, s * nl, nl)
        uk, uv = W.update_batch(cfg, keys, s * nu, nu) if nu else (None, None)
        t0 = time.perf_counter()
        o.lookup(q)
        if nu:
            o.update(uk, uv)
        dt = time.perf_counter() - t0
        if s >= args.warmup:
            times.append(dt)
    ms = 1e3 * float(np.mean(times))
    val = (nl + nu) / (ms * 1e-3) / 1e6
    line = {"impl": "reference", "metric": METRIC, "value": round(val, 3), "unit": "Mops/s",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 3),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": {"u64": "u64", "u32": "u32", "bytes": "u8[32]"}[cfg.kind],
            "data": "synthetic (seeded splitmix64, SURVEY §8(d) recipe)",
            "config": {"workload": f"{args.config}: {cfg.description}", "sample_per_step":
                       {"lookups": nl, "updates": nu}},
            "cpu_baseline": {"value": round(val, 3), "unit": "Mops/s", "cores": 1, "kind": "oracle",
                             "sample": f"{nl} lookups + {nu} updates per step of the {args.config} stream, "
                                       f"pointer-ART oracle built over all {keys.shape[0]} keys "
                                       f"({build_s:.1f} s, untimed)"},
            "e2e": {"value": round(val, 3), "unit": "Mops/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ inputs
def make_keys(cfg, dev):
    """(host keys, host values, device keys) of the config's build set."""
    import torch
    c = W.config_id(cfg)
    vals = W.values_for(W.SEED_VALUES + c, np.arange(cfg.n_keys, dtype=np.uint64))
    if cfg.kind == "u64":
        keys_d = W.u64_keys_torch(c, cfg.n_keys, dev)
        return keys_d.cpu().numpy().view(np.uint64), vals, keys_d
    if cfg.kind == "u32":
        keys = np.arange(cfg.n_keys, dtype=np.uint32)
        return keys, vals, torch.from_numpy(keys.view(np.int32)).to(dev)
    slots, lens = W.string_keys(c, cfg.n_keys)
    return (slots, lens), vals[: lens.shape[0]], (torch.from_numpy(slots).to(dev), torch.from_numpy(lens).to(dev))


def make_lookups(cfg, keys_d, start, m, dev):
    if cfg.kind == "bytes":
        return W.string_lookup_torch(cfg, keys_d[0], keys_d[1], start, m)
    return W.lookup_batch_torch(cfg, keys_d, start, m, device=dev)


# ------------------------------------------------------------------ config 5 (mixed rounds, partitioned)
def c5_local_keys(world, rank, dev, chunk=1 << 27):
    """This rank's share of the 2^30 c5 keys under uniform splitters r*2^64/P (P a
    power of two: owner = top log2(P) key bits; balanced for uniform random keys)."""
    import torch
    c, n = 5, W.C5.n_keys
    bits = world.bit_length() - 1
    ks, vs = [], []
    for s0 in range(0, n, chunk):
        idx = torch.arange(s0, min(n, s0 + chunk), dtype=torch.int64, device=dev)
        k = W.splitmix64_torch(W.SEED_KEYS + c, idx)
        mine = (W._t_srl(k, 64 - bits) == rank) if bits else torch.ones_like(k, dtype=torch.bool)
        v = W.splitmix64_torch(W.SEED_VALUES + c, idx[mine])
        v = torch.where(v == -1, torch.zeros_like(v), v)
        ks.append(k[mine].cpu())
        vs.append(v.cpu())
    splitters = np.array([(r << (64 - bits)) for r in range(1, world)], dtype=np.uint64) if bits else np.zeros(0, np.uint64)
    return torch.cat(ks).numpy().view(np.uint64), torch.cat(vs).numpy().view(np.uint64), splitters


def hbm_peak():
    """(GB/s, source): MEASURED_PEAKS.json hbm_gbs, else the profiling guide's fallback."""
    peaks_path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(peaks_path):
        with open(peaks_path) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md)"


def tree_bytes_touched(stats, hits):
    """Estimated compulsory DRAM bytes of the tree a batch reads once: every inner
    node (a uniform batch of this size reaches all of them) plus the leaves the hits
    touch (1 - exp(-hits / leaves) of them: uniform picks with replacement)."""
    inner = sum(stats[t + "_bytes"] for t in ("n4", "n16", "n48", "n256"))
    leaves = stats["leaf8"] + stats["leaf16"] + stats["leaf32"]
    leaf_b = sum(stats[t + "_bytes"] for t in ("leaf8", "leaf16", "leaf32"))
    frac = 1.0 - float(np.exp(-hits / max(1, leaves)))
    return inner + leaf_b * frac, frac


def run_c5(args, world, rank, local, dev):
    """A step = one round of the mixed stream: this rank's 1/P slice of 2^29 global ops
    (strong scaling: the round is fixed), lookups then updates (reading C7).

    --c5-share P (one GPU): the per-GPU share of a P-GPU run -- rank 0's key range
    (byte0 in [0, 256/P): 2^30 / P keys) and the round's ops that rank 0 owns (~2^29/P),
    served by the same multi-GPU layer at one rank (no exchange: the local part of
    what every GPU of the P-GPU run does per round)."""
    import torch
    import torch.distributed as dist

    import paper_conf_icpp_koppehelggp21_b200 as C
    from paper_conf_icpp_koppehelggp21_b200.dist import DistIndex
    if world & (world - 1):
        raise SystemExit("c5 needs a power-of-two GPU count")
    share = args.c5_share if world == 1 else 0
    if share and share & (share - 1):
        raise SystemExit("--c5-share needs a power of two")
    t0 = time.perf_counter()
    keys, vals, sp = c5_local_keys(share or world, rank, dev)
    di = DistIndex(keys, vals, mode="range", transport=args.transport, lut_bytes=args.lut,
                   splitters=sp if world > 1 else None, keys_local=world > 1, rank=rank, world=world)
    build_s = time.perf_counter() - t0
    stats = di.index.stats()
    R, per = W.C5_ROUND, W.C5_ROUND // world
    rounds = []
    for r in range(2):
        k, u, v = W.mixed_ops_torch(5, W.C5.n_keys, r * R + rank * per, per, dev)
        if share:                                   # rank 0's ops of the round (top log2(P) key bits = 0)
            mine = W._t_srl(k, 64 - (share.bit_length() - 1)) == 0
            k, u, v = k[mine].contiguous(), u[mine].contiguous(), v[mine].contiguous()
        rounds.append((k, u, v))
    torch.cuda.synchronize()
    stream = torch.cuda.current_stream()
    n_ops = int(sum(r[0].shape[0] for r in rounds) // 2)
    n_look = int(sum(int((r[1] == 0).sum().item()) for r in rounds) // len(rounds))

    def step(i, ev=None):
        k, u, v = rounds[i % 2]
        di.mixed_round(k, v, u, events=ev, fused=args.c5_fused == 1)

    for i in range(args.warmup):
        step(i)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(5)] for _ in range(args.steps)]
    clocks = ClockSampler(local)
    clocks.start()
    time.sleep(0.3)
    launches0 = C.cuart_launch_count()
    t_start = torch.cuda.Event(enable_timing=True)
    t_end = torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    C.cuart_kernel_timer(di.h, True)           # CUDA events around every owner walk launch
    t_start.record(stream)
    for i in range(args.steps):
        step(i, evs[i])
    t_end.record(stream)
    torch.cuda.synchronize()
    launches = C.cuart_launch_count() - launches0
    ktot, klaunch, kq, _ = C.cuart_kernel_time_ex(di.h)
    C.cuart_kernel_timer(di.h, False)
    if world > 1:
        dist.barrier()
    clk = clocks.stop()
    if args.c5_fused:        # one cuart_dist_mixed call: only its total is bracketed
        phases = [0.0, float(np.mean([e[0].elapsed_time(e[4]) for e in evs])), 0.0, 0.0]
    else:
        phases = [float(np.mean([e[p].elapsed_time(e[p + 1]) for e in evs])) for p in range(4)]
    tt = torch.tensor([t_start.elapsed_time(t_end), ktot / args.steps] + phases, dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
    total_ms, kern_ms, part_ms, look_ms, upd_ms, unr_ms = tt.tolist()
    ms_step = total_ms / args.steps
    value = (world * n_ops if share == 0 else n_ops) / (ms_step * 1e-3) / 1e6
    peak, peak_src = hbm_peak()
    served = kq / max(1, args.steps)                  # lookups this rank's owner walks served per step
    tree_b, leaf_frac = tree_bytes_touched(stats, served * 0.5)
    bpl = 16.0 + tree_b / max(1.0, served)            # key in + result out + the tree read once per round
    achieved = bpl * served / (kern_ms * 1e-3) / 1e9
    traffic = None
    tfile = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tfile):
        with open(tfile) as f:
            traffic = json.load(f).get(f"c5{'_share' + str(share) if share else ''}/walk")
    if rank == 0:
        print(json.dumps({
            "metric": METRIC, "value": round(value, 3), "unit": "Mops/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms_step, 4), "higher_is_better": True,
            "scaling": "strong" if not share else "share",
            "vs_baseline": None, "dtype": "u64",
            "data": "synthetic (seeded splitmix64, SURVEY §8(d) c5 recipe)",
            "config": {"workload": f"c5: {W.C5.description}" + (f" -- per-GPU share of a {share}-GPU run" if share else ""),
                       "keys": W.C5.n_keys, "round_ops": R, "ops_per_rank_per_step": n_ops,
                       "lookups_per_rank_per_step": n_look, "update_fraction": W.C5_UPDATE_P, "mode": "range",
                       "transport": args.transport, "parallelism": f"range{world}" if not share else f"share-of-{share}",
                       "local_keys_rank0": int(keys.shape[0]), "build_s": round(build_s, 2),
                       "lut_format": stats["lut_format"], "tree_bytes": int(sum(stats[t + "_bytes"] for t in (
                           "n4", "n16", "n48", "n256", "leaf8", "leaf16", "leaf32")))},
            "phases_ms": ({"dist_mixed (lookup pass + update pass)": round(look_ms, 4)} if args.c5_fused else
                          {"partition_by_flag": round(part_ms, 4), "dist_lookup": round(look_ms, 4),
                           "dist_update": round(upd_ms, 4), "unroute": round(unr_ms, 4)}),
            "lookup": None if args.c5_fused else {
                "mlookups_per_s": round(world * n_look / (look_ms * 1e-3) / 1e6, 3), "ms": round(look_ms, 4)},
            "update": None if args.c5_fused else {
                "mupdates_per_s": round(world * (n_ops - n_look) / (upd_ms * 1e-3) / 1e6, 3), "ms": round(upd_ms, 4)},
            "roofline": {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                         "frac": round(achieved / peak, 4), "traffic": traffic,
                         "kernel": ("k_lookup_wq<KeyU64>" if stats.get("wide_lut") else "k_lookup<KeyU64>")
                         + " (owner walk of the multi-GPU layer, fused return)",
                         "kernel_ms": round(kern_ms, 4), "lookups_per_step": int(served),
                         "launches_per_step": round(klaunch / max(1, args.steps), 2),
                         "bytes_per_lookup": round(bpl, 3),
                         "bytes_model": "key in + result out (16 B) + the tree read once per round: every inner "
                                        f"node + the touched fraction of the leaves ({leaf_frac:.3f} for "
                                        f"{int(served * 0.5)} hits)",
                         "peak_source": peak_src},
            "e2e": None, "cpu_baseline": None, "gpu_launches": int(launches), "clocks": clk}), flush=True)
    di.close()
    if world > 1:
        dist.destroy_process_group()


# ------------------------------------------------------------------ main (GPU)
LUT_FORMATS = {"auto": 0, "links": 1, "compact32": 2, "rank": 3}


def main():
    args = _args()
    if args.impl == "reference":
        run_reference(args)
        return
    import torch
    import torch.distributed as dist

    import paper_conf_icpp_koppehelggp21_b200 as C
    from paper_conf_icpp_koppehelggp21_b200.dist import DistIndex

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0")) % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        # NCCL over NVLink/NVSwitch; CUART_DIST_BACKEND=gloo only to smoke-test the
        # multi-rank path with several ranks sharing one GPU (host-staged collectives)
        backend = os.environ.get("CUART_DIST_BACKEND", "nccl")
        dist.init_process_group(backend, device_id=dev if backend == "nccl" else None)
    mode = "single" if world == 1 and not args.dist else args.mode
    if args.config == "c5":
        run_c5(args, world, rank, local, dev)
        return

    cfg = W.CONFIGS[args.config]
    t0 = time.perf_counter()
    keys, vals, keys_d = make_keys(cfg, dev)
    if world == 1 and not args.dist:
        layout = C.Layout(keys, vals, lut_bytes=args.lut)
        ix = C.Index.from_layout(layout, device=local, lut_format=LUT_FORMATS[args.lut_format], skip_log2=args.skip_log2,
                                 l2_persist=args.l2_persist)
        di = None
    else:
        di = DistIndex(keys, vals, mode=mode, transport=args.transport, lut_bytes=args.lut, rank=rank, world=world)
        ix = di.index
        layout = None
    build_s = time.perf_counter() - t0
    stats = ix.stats()

    # resident inputs: this rank's shard of the global lookup stream and update stream
    nl = cfg.n_lookups
    q = make_lookups(cfg, keys_d, rank * nl, nl, dev)
    out = torch.empty(nl, dtype=torch.int64, device=dev)
    q_bytes = sum(t.numel() * t.element_size() for t in q) if isinstance(q, tuple) else q.numel() * q.element_size()
    nu = cfg.n_updates
    uk = uv = None
    if nu:
        uk, uv = W.update_batch_torch(cfg, keys_d, rank * nu, nu)
    torch.cuda.synchronize()

    # algorithmic bytes of the dominant kernel (k_lookup): exact sector count of the
    # lookup path over this rank's layout for a 2^20-query sample + key-in/value-out
    from paper_conf_icpp_koppehelggp21_b200.dist import owners, prefix8, select
    if layout is None:
        local_keys = keys if mode == "replica" else select(keys, owners(prefix8(keys), di.splitters) == rank)
        nloc = local_keys[1].shape[0] if isinstance(local_keys, tuple) else local_keys.shape[0]
        layout = C.Layout(local_keys, np.zeros(nloc, np.uint64), lut_bytes=args.lut)
    if isinstance(q, tuple):
        samp = (q[0][: 1 << 20].cpu().numpy(), q[1][: 1 << 20].cpu().numpy())
    else:
        samp = q[: 1 << 20].cpu().numpy()
        samp = samp.view(np.uint64) if cfg.kind == "u64" else samp.view(np.uint32)
    if mode == "range":   # sample of the queries this rank's index actually serves
        samp = select(samp, owners(prefix8(samp), di.splitters) == rank)
    bucketed = nl >= (1 << 22) and cfg.kind != "bytes" and os.environ.get("CUART_PREBUCKET", "1") != "0"
    # the bucketed wide walk over integer keys runs as k_lookup_wq (2 queries per thread)
    wq = bucketed and bool(stats.get("wide_lut", 0)) and os.environ.get("CUART_ILP", "2") != "1"
    # sectors of the path the walk kernel takes: the pre-bucketed walk starts from the
    # wide root table when the index has one (stats["wide_lut"]), else the plain path
    sec = layout.sectors(samp, wide=bool(bucketed and stats.get("wide_lut", 0)),
                         skip_prefix=int(stats.get("skip_prefix", 0))).astype(np.float64)
    io_bytes = {"u64": 8, "u32": 4, "bytes": 33}[cfg.kind] + 8
    random_bytes_per_lookup = 32.0 * sec.mean() + io_bytes
    # tile form of K-BUCKET (cuart_build_opts.bucket_form, default): single-index integer
    # lookups; the multi-GPU owner walks (fused return) keep the global form
    tile = bucketed and di is None and os.environ.get("CUART_BUCKET_FORM", "2") != "1" and \
        os.environ.get("CUART_SLICE", "0") != "2"
    # whole lookup call, streaming bytes per query: global form = histogram + scatter +
    # walk I/O + gather; tile form = tile sort + walk I/O + tile gather (run padding,
    # ~2%, not counted)
    ks = io_bytes - 8
    if tile:
        stream_bytes = (ks + ks + 2) + (ks + 8) + (8 + 2 + 8)
    else:
        stream_bytes = (ks + (ks + ks + 2) + (ks + 8) + (8 + 2 + 8)) if bucketed else io_bytes
    del samp

    stream = torch.cuda.current_stream()

    def step(ev=None, kev=None):
        if ev is not None:
            ev[0].record(stream)
        if di is None:
            if kev is not None:
                kev[0].record(stream)
            ix.lookup(q, out, stream)
            if kev is not None:
                kev[1].record(stream)
        else:
            di.lookup(q, out)
        if ev is not None:
            ev[1].record(stream)
        if nu:
            if di is None:
                ix.update(uk, uv, stream)
            else:
                di.update(uk, uv)
        if ev is not None:
            ev[2].record(stream)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(args.steps)]
    clocks = ClockSampler(local)
    clocks.start()
    time.sleep(0.3)
    launches0 = C.cuart_launch_count()
    torch.cuda.synchronize()
    C.cuart_kernel_timer(ix.h, True)           # CUDA events around every k_lookup launch
    t_start = torch.cuda.Event(enable_timing=True)
    t_end = torch.cuda.Event(enable_timing=True)
    t_start.record(stream)
    for s in range(args.steps):
        step(evs[s])
    t_end.record(stream)
    torch.cuda.synchronize()
    launches = C.cuart_launch_count() - launches0
    if world > 1:
        dist.barrier()
    clk = clocks.stop()
    total_ms = t_start.elapsed_time(t_end)
    look_ms = float(np.mean([e[0].elapsed_time(e[1]) for e in evs]))
    upd_ms = float(np.mean([e[1].elapsed_time(e[2]) for e in evs])) if nu else 0.0
    ktot, klaunch, kq, kslice = C.cuart_kernel_time_ex(ix.h)
    C.cuart_kernel_timer(ix.h, False)
    kern_ms = ktot / args.steps                # the walk's time per step (every launch of the step)
    served = kq / args.steps                   # lookups the walk served per step
    launches_per_step = klaunch / args.steps
    tt = torch.tensor([total_ms, look_ms, upd_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
    total_ms, look_ms, upd_ms = tt.tolist()
    ms_step = total_ms / args.steps
    # whole job: every rank's lookups + every rank's update ops (each op counted once)
    ops_per_step = world * nl + world * nu
    value = ops_per_step / (ms_step * 1e-3) / 1e6

    out_now = out if di is None else di.lookup(q, out)
    hit = float((out_now[: 1 << 24] != -1).float().mean().item())
    del out_now
    # Algorithmic (compulsory) DRAM bytes of the dominant kernel, the walk (
    # S_DRAM excludes what is L2-resident by construction): key in + result
    # out, plus every tree record the batch needs read once -- all inner nodes and the
    # touched fraction of the leaves.  ncu's measured DRAM bytes ("traffic") above this
    # are re-reads the walk's access order causes.
    tree_b, leaf_frac = tree_bytes_touched(stats, served * hit)
    bytes_per_lookup = io_bytes + tree_b / max(1.0, served)
    pipeline_bytes = stream_bytes + tree_b / max(1.0, served)
    peak, peak_src = hbm_peak()
    achieved = served * bytes_per_lookup / (kern_ms * 1e-3) / 1e9
    pipe_achieved = nl * pipeline_bytes / (look_ms * 1e-3) / 1e9
    # BASELINE north_star's definition: 32-B sectors touched per query x queries/s
    # (the whole lookup call) against peak DRAM bandwidth
    ns_achieved = nl * random_bytes_per_lookup / (look_ms * 1e-3) / 1e9
    traffic = args.traffic
    tfile = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if traffic is None and os.path.exists(tfile):
        with open(tfile) as f:
            traffic = json.load(f).get(f"{args.config}/{'tile' if tile else 'bucketed' if bucketed else 'direct'}")

    # end-to-end through the public API with HOST buffers (pinned), copies inside the timed region
    e2e = None
    if not args.no_e2e:
        def pinned(t):
            h = torch.empty(t.shape, dtype=t.dtype, pin_memory=True)
            h.copy_(t)
            return h

        qh = tuple(pinned(t) for t in q) if isinstance(q, tuple) else pinned(q)
        qn = tuple(t.numpy() for t in qh) if isinstance(qh, tuple) else qh.numpy()
        qbytes = sum(t.numel() * t.element_size() for t in qh) if isinstance(qh, tuple) else qh.numel() * qh.element_size()
        oh = torch.empty(nl, dtype=torch.int64, pin_memory=True)
        ukh = uvh = None
        if nu:
            ukh = torch.empty(uk.shape[0], dtype=torch.int64, pin_memory=True)
            uvh = torch.empty_like(ukh)
            ukh.copy_(uk)
            uvh.copy_(uv)

        def e2e_step():
            if di is None:
                C.cuart_lookup_host(ix.h, qn, oh.numpy())
                if nu:
                    C.cuart_update_host(ix.h, ukh.numpy(), uvh.numpy())
            else:
                qd = tuple(t.to(dev, non_blocking=True) for t in qh) if isinstance(qh, tuple) else qh.to(dev, non_blocking=True)
                oh.copy_(di.lookup(qd, out), non_blocking=True)
                if nu:
                    di.update(ukh.to(dev, non_blocking=True), uvh.to(dev, non_blocking=True))
                torch.cuda.synchronize()

        e2e_step()
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        ts = []
        for _ in range(args.e2e_steps):
            t0 = time.perf_counter()
            e2e_step()
            ts.append(time.perf_counter() - t0)
        et = torch.tensor([float(np.mean(ts))], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(et, op=dist.ReduceOp.MAX)
        e_s = et.item()
        e2e = {"value": round(ops_per_step / e_s / 1e6, 3), "unit": "Mops/s",
               "h2d_bytes_per_step": int(qbytes + nu * 16), "d2h_bytes_per_step": int(nl * 8),
               "ms_per_step": round(e_s * 1e3, 3),
               "api": ("cuart_lookup_host + cuart_update_host (pinned host buffers, chunked H2D/kernel/D2H)"
                       if di is None else "pinned H2D + DistIndex.lookup/update + D2H")}
        del qh, qn, oh, ukh, uvh

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        nls = min(nl, 1 << 22)
        nus = min(nu, nls * nu // nl) if nu else 0
        v, det = oracle_timing(cfg, keys, vals, nls, nus)
        cpu = {"value": round(v, 3), "unit": "Mops/s", "cores": 1, "kind": "oracle",
               "sample": f"{nls} lookups + {nus} updates of the {args.config} stream (same mix), "
                         f"single-threaded pointer ART built over all {cfg.n_keys} keys, pinned to one core "
                         f"(build {det['build_s']} s untimed, timed {det['seconds']} s); all-core lookups: "
                         f"{det['allcore_sample_lookups']} further lookups over {det['host_cores']} threads",
               **{k: det[k] for k in ("oracle_lookup_mops_1core", "oracle_update_mops_1core",
                                      "oracle_lookup_mops_allcores", "host_cores")}}
        if layout is not None:
            cpu["f3_layout_engine"] = layout_engine_timing(cfg, keys, layout, nls, det)

    if rank == 0:
        line = {
            "metric": METRIC, "value": round(value, 3), "unit": "Mops/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_step, 4),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": {"u64": "u64", "u32": "u32", "bytes": "u8[32]"}[cfg.kind],
            "data": "synthetic (seeded splitmix64 keys/queries/updates, SURVEY §8(d) recipe)",
            "config": {"workload": f"{args.config}: {cfg.description}", "keys": cfg.n_keys,
                       "lookups_per_rank": nl, "updates_per_rank": nu, "key_kind": cfg.kind,
                       "lut_bytes": args.lut, "lut_format": stats["lut_format"], "mode": mode,
                       "skip_table": {"prefix_bytes": stats.get("skip_prefix", 0), "slots": stats.get("skip_slots", 0)},
                       "transport": args.transport if (world > 1 or args.dist) and mode == "range" else None,
                       "parallelism": f"{mode}{world}" if world > 1 or args.dist else "single",
                       "l2": f"inputs ({q_bytes / 2**30:.1f} GiB of queries per step) larger than L2; no flush",
                       "measured_hit_ratio": round(hit, 4), "build_s": round(build_s, 2)},
            "lookup": {"mlookups_per_s": round(world * nl / (look_ms * 1e-3) / 1e6, 3), "ms": round(look_ms, 4)},
            "update": {"mupdates_per_s": round(world * nu / (upd_ms * 1e-3) / 1e6, 3) if nu else None,
                       "ms": round(upd_ms, 4)},
            "roofline": {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                         "frac": round(achieved / peak, 4), "traffic": traffic,
                         "kernel": ("k_lookup_slice" if kslice else "k_lookup_wt" if tile else "k_lookup_wq" if wq
                                    else "k_lookup")
                         + {"u64": "<KeyU64>", "u32": "<KeyU32>", "bytes": "<KeyBytes>"}[cfg.kind],
                         "kernel_ms": round(kern_ms, 4), "lookups_per_step": int(served),
                         "launches_per_step": round(launches_per_step, 2),
                         "lookup_call_ms": round(look_ms, 4), "prebucket": "on" if bucketed else "off",
                         "bytes_per_lookup": round(bytes_per_lookup, 3),
                         "bytes_model": "compulsory: key in + result out + every inner node and the touched "
                                        f"fraction of the leaves ({leaf_frac:.3f}) read once per batch",
                         "sectors_per_lookup": round(float(sec.mean()), 4),
                         "random_path_bytes_per_lookup": round(random_bytes_per_lookup, 3),
                         "peak_source": peak_src, "random_access_ceiling": RANDOM_CEILING,
                         "north_star_random_sector": {
                             "definition": "BASELINE north_star: 32-B sectors touched per query (host walker over "
                                           "the kernel's path, 2^20-query sample) x 32 B + key/result I/O, times "
                                           "lookups/s of the whole lookup call, vs peak DRAM bandwidth",
                             "sectors_per_lookup": round(float(sec.mean()), 4),
                             "bytes_per_lookup": round(random_bytes_per_lookup, 3),
                             "achieved": round(ns_achieved, 1), "frac": round(ns_achieved / peak, 4)},
                         "lookup_call": {"ms": round(look_ms, 4), "bytes_per_lookup": round(pipeline_bytes, 3),
                                         "achieved": round(pipe_achieved, 1), "frac": round(pipe_achieved / peak, 4),
                                         "kernels": "k_tsort, k_lookup_wt, k_tgather" if tile else
                                         "k_bhist, k_bscan_rows, k_bscan, k_bscatter, "
                                         + ("k_lookup_slice" if kslice else "k_lookup_wq" if wq else "k_lookup") + ", k_bgather"
                                         if bucketed else "k_lookup"}},
            "e2e": e2e, "cpu_baseline": cpu, "gpu_launches": int(launches), "clocks": clk,
            "index": {k: stats[k] for k in ("n4", "n16", "n48", "n256", "leaf8", "arena_bytes", "max_depth",
                                            "lut_exceptions")},
        }
        print(json.dumps(line), flush=True)
    if di is not None:
        di.close()
    else:
        ix.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
