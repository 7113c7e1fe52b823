import csv, sys, subprocess, io
rep, kname = sys.argv[1], sys.argv[2]
thr = float(sys.argv[3]) if len(sys.argv) > 3 else 0.004
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass",
                      "-k", f"regex:{kname}"], capture_output=True, text=True).stdout
lines = out.splitlines()
# may contain multiple kernels; take first table
start = [i for i, l in enumerate(lines) if l.startswith('"Address"')]
rows = list(csv.reader(lines[start[0]:]))
h = rows[0]
ix = {k: i for i, k in enumerate(h)}
data = [r for r in rows[1:] if len(r) == len(h)]
S = "Warp Stall Sampling (All Samples)"
tot = sum(int(r[ix[S]] or 0) for r in data)
print("total samples", tot, "instrs", len(data))
stall_cols = [k for k in h if k.startswith("stall_") or "Stall Reasons" in k]
for r in data:
    s = int(r[ix[S]] or 0)
    ex = int(r[ix["Instructions Executed"]] or 0)
    if s > tot * thr:
        print(f'{r[0][-5:]} ex={ex:>8} smp={s:>5} {100*s/tot:5.1f}%  {r[1][:80]}')
