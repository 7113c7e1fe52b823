"""Per-CTA phase timeline of one one-pass offset-branch launch (needs a
-DDEFCON_PROBE_OP_TIMELINE build: python tools/build_variants.py optl=-DDEFCON_PROBE_OP_TIMELINE).

  DEFCON_LIB=tools/bin/libdefcon_optl.so python tools/op_timeline.py [config]
Stamps (globaltimer ns, relative to the earliest CTA start): 0 start, 1 setup, 2 after griddep,
4+2k chunk k x-stage ready, 5+2k chunk k barrier passed, 20 loop end, 21 last MMA done, 22 epilogue end.
"""
import ctypes
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from defcon_workloads import configs, inputs  # noqa: E402
import paper_conf_ipps_jayaweeralwrk24_b200 as d  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "yolact_r101_c4_v2"
c = configs.SINGLE_LAYER[name]
lib = d.load_library()
dev = torch.device("cuda")
x = torch.from_numpy(inputs.gen_x(c)).to(dev, torch.bfloat16)
P = {k: torch.from_numpy(v).to(dev) for k, v in inputs.gen_offset_branch(c).items()}
for _ in range(3):
    d.defcon_offset_dw_conv(x, P["dw_w"], P["dw_scale"], P["dw_shift"], P["pw_w"], P["pw_b"], offset_groups=c.G)
torch.cuda.synchronize()
buf = np.zeros((1024, 48), dtype=np.uint64)
lib.defcon_debug_op_timeline(buf.ctypes.data_as(ctypes.c_void_p))
grid = int((buf[:, 0] > 0).sum())
b = buf[:grid].astype(np.int64)
t0 = b[:, 0].min()
r = np.where(b > 0, b - t0, -1)
print(f"{name}: grid {grid}, kernel span {(b.max() - t0) / 1e3:.2f} us")
names = {0: "start", 1: "setup", 2: "griddep"}
for k in range(8):
    names[4 + 2 * k] = f"x{k} ready"
    names[5 + 2 * k] = f"bar{k}"
for k in range(3, 8):
    names[32 + k] = f"ld{k} issued"
for k in range(8):
    names[40 + k] = f"mma{k} go"
names.update({20: "loop end", 21: "mma done", 22: "epi end", 24: "k3 top", 25: "k3 A free", 26: "epi ld0 beg",
              27: "epi ld0 end", 28: "epi pre", 29: "epi cb0 done", 23: "epi staged", 30: "epi bar", 31: "dealloc"})
for i, nm in names.items():
    v = r[:, i]
    v = v[v >= 0]
    if len(v):
        print(f"  {nm:10s} n={len(v):4d} min {v.min()/1e3:7.2f} med {np.median(v)/1e3:7.2f} max {v.max()/1e3:7.2f} us")
