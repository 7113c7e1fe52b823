"""Host<->device copy rates on this box: H2D alone, D2H alone, both at once on two streams
(pinned host buffers, CUDA events).  python tools/probe_pcie.py [MiB]"""
import sys

import torch

mb = int(sys.argv[1]) if len(sys.argv) > 1 else 10
n = mb << 20
h1 = torch.empty(n, dtype=torch.uint8).pin_memory()
h2 = torch.empty(n, dtype=torch.uint8).pin_memory()
d1 = torch.empty(n, dtype=torch.uint8, device="cuda")
d2 = torch.empty(n, dtype=torch.uint8, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def timed(fn, reps=20):
    fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps


def both():
    cur = torch.cuda.current_stream()
    s1.wait_stream(cur)
    s2.wait_stream(cur)
    with torch.cuda.stream(s1):
        d1.copy_(h1, non_blocking=True)
    with torch.cuda.stream(s2):
        h2.copy_(d2, non_blocking=True)
    cur.wait_stream(s1)
    cur.wait_stream(s2)


for _ in range(3):
    t_h2d = timed(lambda: d1.copy_(h1, non_blocking=True))
    t_d2h = timed(lambda: h2.copy_(d2, non_blocking=True))
    t_both = timed(both)
print(f"{mb} MiB: H2D {t_h2d*1e3:.1f} us ({n/t_h2d/1e6:.1f} GB/s), D2H {t_d2h*1e3:.1f} us ({n/t_d2h/1e6:.1f} GB/s), "
      f"both concurrently {t_both*1e3:.1f} us")
