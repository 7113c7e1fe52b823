#!/bin/bash
# Run on the GPU box (via gpurun) from the repo root: bench line + ncu launch list + one
# `ncu --set full` capture of each hot-path kernel, summaries written under gpurun_out/.
set -u
R=${1:-r01}
mkdir -p gpurun_out
python paper_conf_ipps_jayaweeralwrk24_b200/build.py > /dev/null 2>&1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/${R}_gpu.txt
python bench.py > gpurun_out/${R}_bench.json 2> gpurun_out/${R}_bench.err
# launch list of the bench command (cold-cache, serialised: compare shares, not absolutes)
ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv \
    --log-file gpurun_out/${R}_launches.csv python bench.py --steps 4 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
# one full capture per hot-path kernel, same command
ncu --set full --clock-control none --import-source on -k regex:"dcn_fwd|dw_bn|pw_" -s 3 -c 3 \
    -o gpurun_out/${R}_full python bench.py --steps 4 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
ncu -i gpurun_out/${R}_full.ncu-rep --page details --csv > gpurun_out/${R}_full_details.csv 2>/dev/null
ncu -i gpurun_out/${R}_full.ncu-rep --page raw --csv > gpurun_out/${R}_full_raw.csv 2>/dev/null
echo done
