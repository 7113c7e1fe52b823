#!/bin/bash
# Per-kernel durations of the offset-branch kernels (warm L2, serialised) + the graph-replay probe.
python paper_conf_ipps_jayaweeralwrk24_b200/build.py >/dev/null 2>&1
ncu --metrics gpu__time_duration.sum,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum --clock-control none --cache-control none -k regex:"${2:-dw_bn|pw_si}" -c 40 --csv python tools/probe_branch.py ${1:-yolact_r101_c4_v2} > gpurun_out/kprof.csv 2>/dev/null
python tools/probe_branch.py
