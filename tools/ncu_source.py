import csv, sys, subprocess
rep, kname = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass",
                      "-k", f"regex:{kname}"], capture_output=True, text=True).stdout
lines = out.splitlines()
start = [i for i, l in enumerate(lines) if l.startswith('"Address"')]
rows = list(csv.reader(lines[start[0]:]))
h = rows[0]
ix = {k: i for i, k in enumerate(h)}
data = [r for r in rows[1:] if len(r) == len(h) and r[0] != "Address"]
seen = set(); data = [r for r in data if not (r[0] in seen or seen.add(r[0]))]
S = "Warp Stall Sampling (All Samples)"
tot = sum(int(r[ix[S]] or 0) for r in data)
stall_cols = [k for k in h if k.startswith("stall_") and "Not Issued" not in k]
print("total samples", tot)
agg = {}
for r in data:
    for k in stall_cols:
        agg[k] = agg.get(k, 0) + int(r[ix[k]] or 0)
print(sorted(agg.items(), key=lambda t: -t[1])[:8])
order = sorted(range(len(data)), key=lambda i: -int(data[i][ix[S]] or 0))[:top]
for i in sorted(order):
    r = data[i]
    s = int(r[ix[S]] or 0)
    st = sorted(((int(r[ix[k]] or 0), k[6:]) for k in stall_cols), reverse=True)[:2]
    print(f'{i:5d} {r[0][-5:]} ex={int(r[ix["Instructions Executed"]] or 0):>8} {100*s/tot:5.1f}% {st[0][1]}:{st[0][0]} {st[1][1]}:{st[1][0]}  {r[1][:70]}')
