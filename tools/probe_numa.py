"""H2D / D2H rates of pinned buffers allocated from the GPU's local NUMA node vs elsewhere."""
import os
import subprocess
import sys

import torch

bdf = subprocess.run(["nvidia-smi", "--query-gpu=pci.bus_id", "--format=csv,noheader"], capture_output=True,
                     text=True).stdout.split()[0].lower()
bdf = bdf[4:] if bdf.count(":") == 2 and len(bdf.split(":")[0]) == 8 else bdf
path = f"/sys/bus/pci/devices/{bdf}"
if not os.path.exists(path):
    cands = [p for p in os.listdir("/sys/bus/pci/devices") if p.endswith(bdf.split(":", 1)[-1])]
    path = "/sys/bus/pci/devices/" + cands[0]
node = open(path + "/numa_node").read().strip()
local = open(path + "/local_cpulist").read().strip()
print("gpu", bdf, "numa_node", node, "local_cpulist", local, "affinity", sorted(os.sched_getaffinity(0))[:8], "...",
      len(os.sched_getaffinity(0)), "cpus")


def parse(cl):
    out = set()
    for part in cl.split(","):
        a, _, b = part.partition("-")
        out.update(range(int(a), int(b or a) + 1))
    return out


def rates(tag):
    n = 10 << 20
    h1 = torch.empty(n, dtype=torch.uint8).pin_memory()
    h2 = torch.empty(n, dtype=torch.uint8).pin_memory()
    h1.fill_(1)
    d1 = torch.empty(n, dtype=torch.uint8, device="cuda")
    res = []
    for fn in (lambda: d1.copy_(h1, non_blocking=True), lambda: h2.copy_(d1, non_blocking=True)):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(20):
            fn()
        b.record()
        torch.cuda.synchronize()
        res.append(n / (a.elapsed_time(b) / 20) / 1e6)
    print(f"{tag}: H2D {res[0]:.1f} GB/s, D2H {res[1]:.1f} GB/s")


torch.cuda.init()
rates("default affinity")
loc = parse(local) & os.sched_getaffinity(0)
if loc:
    os.sched_setaffinity(0, loc)
    rates(f"pinned to {len(loc)} GPU-local cpus")
other = os.sched_getaffinity(0) if not loc else (set(range(os.cpu_count())) - parse(local))
