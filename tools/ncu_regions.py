"""Instruction mix of one kernel in an ncu report: executed warp-instructions per opcode, and per
contiguous SASS region split at BAR.SYNC (python tools/ncu_regions.py rep kernel_regex)."""
import collections
import csv
import subprocess
import sys

rep, kname = sys.argv[1], sys.argv[2]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass", "-k",
                      f"regex:{kname}"], capture_output=True, text=True).stdout
lines = out.splitlines()
start = [i for i, l in enumerate(lines) if l.startswith('"Address"')]
rows = list(csv.reader(lines[start[0]:]))
h = rows[0]
ix = {k: i for i, k in enumerate(h)}
seen = set()
data = [r for r in rows[1:] if len(r) == len(h) and r[0] != "Address" and not (r[0] in seen or seen.add(r[0]))]
E = ix["Instructions Executed"]
S = ix["Warp Stall Sampling (All Samples)"]
tot = sum(int(r[E] or 0) for r in data)
print("total warp instructions", tot)
ops = collections.Counter()
for r in data:
    t = r[1].split()
    op = t[1] if t[0].startswith("@") else t[0]
    ops[op.split(".")[0]] += int(r[E] or 0)
print(ops.most_common(20))
reg, cur, cnt, smp = [], 0, 0, 0
for i, r in enumerate(data):
    cnt += int(r[E] or 0)
    smp += int(r[S] or 0)
    if "BAR.SYNC" in r[1] or i == len(data) - 1:
        reg.append((cur, i, cnt, smp))
        cur, cnt, smp = i + 1, 0, 0
for a, b, c, s in reg:
    print(f"lines {a:5d}-{b:5d}: {c:>10} instr  {s:>6} samples")
