"""Per-CTA phase timeline of one fused DCN launch (needs a -DDEFCON_PROBE_TIMELINE build).

  DEFCON_LIB=tools/bin/libdefcon_tl.so python tools/timeline.py [config]
Stamps (globaltimer ns, relative to the earliest CTA start): 0 start, 1 setup done,
2+2o / 3+2o producer segment o begin / end, 10/11 metadata table ready, 12/13 last
epilogue begin/end, 14 MMA issuer done, 15 exit.
"""
import ctypes
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from defcon_workloads import configs  # noqa: E402
import paper_conf_ipps_jayaweeralwrk24_b200 as d  # noqa: E402
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from probe_dcn import time_cfg  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "yolact_r101_c4_v2"
c = configs.SINGLE_LAYER[name]
lib = d.load_library()
us, tf = time_cfg(c, "ldg", reps=50)
buf = np.zeros((256, 16), dtype=np.uint64)
lib.defcon_debug_timeline(buf.ctypes.data_as(ctypes.c_void_p))
grid = int((buf[:, 0] > 0).sum())
b = buf[:grid].astype(np.int64)
t0 = b[:, 0].min()
r = np.where(b > 0, b - t0, -1)
print(f"{name}: {us:.2f} us/launch (graph), grid {grid}")
names = {0: "start", 1: "setup", 2: "seg0 beg", 3: "seg0 end", 4: "seg1 beg", 5: "seg1 end", 6: "seg2 beg|fastpath",
         7: "seg2 end|staged", 8: "fix done", 9: "slowpath", 10: "meta0 rdy", 11: "metaN rdy", 12: "epi beg", 13: "epi end", 14: "mma done",
         15: "exit"}
for i, nm in names.items():
    v = r[:, i]
    v = v[v >= 0]
    if len(v):
        print(f"  {nm:10s} n={len(v):3d} min {v.min()/1e3:7.2f} med {np.median(v)/1e3:7.2f} max {v.max()/1e3:7.2f} us")
