"""PCIe probe: pinned host <-> device copy bandwidth alone and concurrent (the
bound of bench.py's e2e leg), GB/s over 4 GiB transfers in 64 MiB chunks."""
import json
import torch

n = 4 << 30
chunk = 64 << 20
h_src = torch.empty(n, dtype=torch.uint8, pin_memory=True)
h_dst = torch.empty(n, dtype=torch.uint8, pin_memory=True)
d_a = torch.empty(n, dtype=torch.uint8, device="cuda")
d_b = torch.empty(n, dtype=torch.uint8, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def run(h2d, d2h):
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    s1.wait_event(e0)
    s2.wait_event(e0)
    for off in range(0, n, chunk):
        if h2d:
            with torch.cuda.stream(s1):
                d_a[off:off + chunk].copy_(h_src[off:off + chunk], non_blocking=True)
        if d2h:
            with torch.cuda.stream(s2):
                h_dst[off:off + chunk].copy_(d_b[off:off + chunk], non_blocking=True)
    ev1, ev2 = s1.record_event(), s2.record_event()
    torch.cuda.current_stream().wait_event(ev1)
    torch.cuda.current_stream().wait_event(ev2)
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / 1e3


for name, a, b in (("h2d", 1, 0), ("d2h", 0, 1), ("both", 1, 1)):
    run(a, b)
    t = min(run(a, b) for _ in range(3))
    print(json.dumps({"probe": name, "seconds": round(t, 4), "GBps_per_direction": round(n / t / 1e9, 2)}), flush=True)
