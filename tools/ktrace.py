"""Per-k-iteration event trace of one CTA of the fused DCN kernel (needs a -DDEFCON_PROBE_KTRACE
build: python tools/build_variants.py kt=-DDEFCON_PROBE_KTRACE).
  DEFCON_LIB=tools/bin/libdefcon_kt.so python tools/ktrace.py [config]
Events (clock64 of CTA KTRACE_CTA, k-iteration q of the CTA): producer thread 0: 0 before empty
wait, 8 / 9 after the lerp + store of row 0 / 1, 10 after the proxy fence, before the arrive; 0 before empty
wait, 1 after it, 2 after its arrive; 7 the last producer warp's arrive; MMA thread: 3 before the
full_a wait, 4 after it, 5 after full_b, 6 after the commit."""
import ctypes
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from defcon_workloads import configs  # noqa: E402
import paper_conf_ipps_jayaweeralwrk24_b200 as d  # noqa: E402
from probe_dcn import time_cfg  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "yolact_r101_c4_v2"
c = configs.SINGLE_LAYER[name]
lib = d.load_library()
us, tf = time_cfg(c, "ldg", reps=20)
buf = np.zeros((24, 64), dtype=np.int64)
lib.defcon_debug_ktrace(buf.ctypes.data_as(ctypes.c_void_p))
n = int((buf[6] > 0).sum())
b = buf[:, :n] - buf[3, 0]
print(f"{name}: {us:.2f} us; {n} k-iterations traced (cycles relative to the first MMA wait)")
for q in range(n):
    if buf[12, q]:
        print(f"segment start at q={q}: sync1 {b[12,q]} -> {b[13,q]}, build -> {b[14,q]}, sync2 -> {b[15,q]}; "
              f"build: enter {b[16,q]} waited {b[17,q]} round done {b[18,q]}; (probe: first build done {b[23,q]})")
print("MMA warp per q: gotB->1st MMA issued, ->last issued, ->commit done, commit->next waitA:",
      [(int(b[16,q]-b[5,q]), int(b[17,q]-b[5,q]), int(b[6,q]-b[5,q]), int(b[3,q+1]-b[6,q]) if q + 1 < n else 0) for q in range(min(n, 12))])
print("MMA serial probe: m:done-m:gotB per q:", [int(b[11,q]-b[5,q]) for q in range(n)] if buf[11].any() else "n/a")
print("  q   p:emptyW  p:got  row0  row1  fence  p0:arr  pLast:arr  m:waitA  m:gotA  m:gotB  m:commit  | MMA period  A-wait  B-wait")
for q in range(n):
    per = b[6, q] - b[6, q - 1] if q else 0
    print(f"{q:3d} {b[0,q]:8d} {b[1,q]:8d} {b[8,q]:5d} {b[9,q]:5d} {b[10,q]:6d} {b[2,q]:8d} {b[7,q]:9d} {b[3,q]:8d} {b[4,q]:8d} {b[5,q]:7d} {b[6,q]:8d}  | {per:6d} {b[4,q]-b[3,q]:6d} {b[5,q]-b[4,q]:6d}")
