"""Count the tcgen05 / TMA / vector-gather / packed-FP32 instructions in each hot-path kernel of
libdefcon.so (cuobjdump -sass), the evidence that the kernels use the sm_100a units.

  python tools/sass_evidence.py > profiles/sass_evidence.txt
"""
import collections
import os
import re
import subprocess

LIB = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                   "paper_conf_ipps_jayaweeralwrk24_b200", "libdefcon.so")
OPS = {  # SASS mnemonic (as the first token of the instruction) -> meaning
    "UTCHMMA": "tcgen05.mma (bf16 / tf32)", "UTCBAR": "tcgen05.commit", "LDTM": "tcgen05.ld",
    "UTMALDG": "TMA load", "UTMASTG": "TMA store", "HMMA": "legacy mma.sync",
    "FFMA2": "packed fp32 FMA", "FFMA": "fp32 FMA", "TEX": "texture fetch",
}
KERNELS = ["dcn_fwd_bf16_tc_kernel", "pw_tc_kernel", "pw_sigmoid_kernel", "dw_bn_relu_kernel",
           "dcn_fwd_f32_tiled_kernel", "deform_columns_rows_kernel", "offset_branch_onepass_kernel",
           "dcn_fwd_simt_kernel"]

sass = subprocess.run(["cuobjdump", "-sass", LIB], capture_output=True, text=True).stdout
stats, cur = collections.OrderedDict(), None
for line in sass.splitlines():
    m = re.search(r"Function : (\S+)", line)
    if m:
        cur = m.group(1)
        stats[cur] = collections.Counter()
        continue
    m = re.search(r"/\*[0-9a-f]{4,}\*/\s+(?:@!?U?P\w+\s+)?([A-Z0-9_]+)(\.[A-Z0-9_.]+)?", line)
    if cur and m:
        op = m.group(1)
        if op in OPS:
            stats[cur][op] += 1
        if op == "LDG" and m.group(2) and ".256" in m.group(2):
            stats[cur]["LDG.256"] += 1
print(f"# {LIB} (cuobjdump -sass), static instruction counts per kernel instantiation")
print("# " + ", ".join(f"{k} = {v}" for k, v in OPS.items()) + ", LDG.256 = 256-bit gather")
for fn, c in stats.items():
    name = next((k for k in KERNELS if k in fn), None)
    if name and c:
        print(f"{fn[:110]:110s}  " + " ".join(f"{k}={v}" for k, v in sorted(c.items())))
