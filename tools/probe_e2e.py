"""Where the end-to-end (host buffers) time goes at the bench workload: the C-ABI host entry
point per call (CUDA events and wall clock), the host-side cost of one call (GPU work skipped by
timing only the Python/C launch path) and the bare copies.  python tools/probe_e2e.py"""
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from defcon_workloads import configs, inputs  # noqa: E402
import paper_conf_ipps_jayaweeralwrk24_b200 as d  # noqa: E402

c = configs.C4
dev = torch.device("cuda")
d.load_library()
x = inputs.gen_x(c)
w, b = inputs.gen_weight(c)
P = {k: torch.from_numpy(v).to(dev) for k, v in inputs.gen_offset_branch(c).items()}
wd, bd = torch.from_numpy(w).to(dev, torch.bfloat16), torch.from_numpy(b).to(dev)
xh = torch.from_numpy(x).to(torch.bfloat16).pin_memory()
yh = torch.empty((c.N, c.Ho, c.Wo, c.Cout), dtype=torch.bfloat16).pin_memory()
for k in (1, 2, 4, 6, 8, 16):
    os.environ["DEFCON_HOST_CHUNKS"] = str(k)
    ws = torch.empty(d.defcon_layer_workspace_size(c.N, c.H, c.W, c.Cin, c.Cout), dtype=torch.uint8, device=dev)
    call = lambda: d.defcon_layer_forward_host(xh, P, wd, bd, yh, ws)
    for _ in range(3):
        call()
    torch.cuda.synchronize()
    a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    a.record()
    for _ in range(20):
        call()
    e.record()
    torch.cuda.synchronize()
    wall = (time.perf_counter() - t0) / 20 * 1e6
    print(f"chunks {k}: {a.elapsed_time(e) / 20 * 1e3:.1f} us/call (events), {wall:.1f} us/call (wall)")
xd = torch.empty(x.shape, dtype=torch.bfloat16, device=dev)
yd = torch.empty(yh.shape, dtype=torch.bfloat16, device=dev)
for _ in range(3):
    xd.copy_(xh, non_blocking=True)
    yh.copy_(yd, non_blocking=True)
torch.cuda.synchronize()
a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
for _ in range(20):
    xd.copy_(xh, non_blocking=True)
    yh.copy_(yd, non_blocking=True)
e.record()
torch.cuda.synchronize()
print(f"bare H2D + D2H (serial, one stream): {a.elapsed_time(e) / 20 * 1e3:.1f} us")

if len(sys.argv) > 1 and sys.argv[1] == "trace":
    from torch.profiler import ProfilerActivity, profile
    for k in (2, 4):
        os.environ["DEFCON_HOST_CHUNKS"] = str(k)
        ws = torch.empty(d.defcon_layer_workspace_size(c.N, c.H, c.W, c.Cin, c.Cout), dtype=torch.uint8, device=dev)
        d.defcon_layer_forward_host(xh, P, wd, bd, yh, ws)
        with profile(activities=[ProfilerActivity.CUDA, ProfilerActivity.CPU]) as prof:
            d.defcon_layer_forward_host(xh, P, wd, bd, yh, ws)
            d.defcon_layer_forward_host(xh, P, wd, bd, yh, ws)
        evs = [e for e in prof.events() if e.device_type.name == "CUDA"]
        evs.sort(key=lambda e: e.time_range.start)
        t0 = evs[0].time_range.start
        print(f"--- chunks {k}: GPU activities of two calls (us from first)")
        for e in evs:
            print(f"{e.time_range.start - t0:9.1f} {e.time_range.end - t0:9.1f}  {e.name[:60]}")
