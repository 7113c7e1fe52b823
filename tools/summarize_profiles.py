"""Summarise an ncu capture + launch list into profiles/<round>_*.md/.json (tracked)."""
import csv
import json
import os
import sys

R = sys.argv[1] if len(sys.argv) > 1 else "r01"
G = "gpurun_out"
P = "profiles"

# launch list
rows = list(csv.reader(open(f"{G}/{R}_launches.csv")))
hdr = None
launch = []
for r in rows:
    if "Kernel Name" in r:
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        launch.append((d["Kernel Name"].split("(")[0].replace("void ", ""), float(d["Metric Value"])))
ours = [(k, v) for k, v in launch if any(s in k for s in ("dcn_fwd", "dw_bn", "pw_", "tex_stage", "offset_branch",
                                                          "op_pack"))]
tot = {}
for k, v in ours:
    tot.setdefault(k, []).append(v)

# full capture
raw = list(csv.reader(open(f"{G}/{R}_full_raw.csv")))
h = raw[0]
want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__throughput.avg.pct_of_peak_sustained_active",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "l1tex__t_sector_hit_rate.pct",
        "lts__t_sector_hit_rate.pct", "smsp__inst_executed.sum"]
units = dict(zip(h, raw[1]))
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-3, "usecond": 1.0,
         "msecond": 1e3}


def val(k, x):
    try:
        v = float(str(x).replace(",", ""))
    except ValueError:
        return x
    u = units.get(k, "")
    if u in SCALE:
        v *= SCALE[u]
    return v


caps = []
for r in raw[2:]:
    d = dict(zip(h, r))
    caps.append({"kernel": d.get("Kernel Name", "").split("(")[0].replace("void ", ""),
                 **{k.replace(".sum", "").replace("gpu__time_duration", "duration_us"): val(k, d.get(k))
                    for k in want}})

summary = {"round": R, "launch_list_us": {k: [round(x / 1000, 2) for x in v] for k, v in tot.items()},
           "full_captures": caps}
dcn = [c for c in caps if "dcn_fwd" in c["kernel"]]
if dcn:
    summary["dcn_dram_bytes_per_launch"] = dcn[0]["dram__bytes_read"] + dcn[0]["dram__bytes_write"]
    summary["dcn_dram_bytes_note"] = (
        "cold: ncu --cache-control all flushes L2 before the replay; y (M x Cout bf16) stays dirty "
        "in the write-back L2 at kernel end, so dram__bytes_write under-counts it")


def extra(name):   # the other captures of the round (columns kernel, fp32 DCN)
    try:
        rr = list(csv.reader(open(f"{G}/{R}_{name}_raw.csv")))
    except OSError:
        return []
    hh, uu = rr[0], dict(zip(rr[0], rr[1]))
    out = []
    for r in rr[2:]:
        d = dict(zip(hh, r))
        rec = {"kernel": d.get("Kernel Name", "").split("(")[0].replace("void ", "")}
        for k in want:
            try:
                v = float(str(d.get(k)).replace(",", "")) * SCALE.get(uu.get(k, ""), 1)
            except (TypeError, ValueError):
                v = d.get(k)
            rec[k.replace(".sum", "").replace("gpu__time_duration", "duration_us")] = v
        out.append(rec)
    return out


summary["columns_capture"] = extra("columns")
summary["f32_3xtf32_capture"] = extra("f32")
json.dump(summary, open(f"{P}/{R}_ncu_summary.json", "w"), indent=1)
print(json.dumps(summary, indent=1)[:3000])
