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
ncu --set full --clock-control none --import-source on -k regex:"dcn_fwd|offset_branch_onepass" -s 4 -c 2 \
    -o gpurun_out/${R}_full python bench.py --steps 4 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
ncu -i gpurun_out/${R}_full.ncu-rep --page details --csv > gpurun_out/${R}_full_details.csv 2>/dev/null
ncu -i gpurun_out/${R}_full.ncu-rep --page raw --csv > gpurun_out/${R}_full_raw.csv 2>/dev/null
# the sampling stage alone (defcon_deform_columns): dram bytes of the columns kernel
ncu --set full --clock-control none -k regex:"deform_columns" -c 1 -o gpurun_out/${R}_columns \
    python tools/probe_sampler.py yolact_r101_c5_v2 > /dev/null 2>&1
ncu -i gpurun_out/${R}_columns.ncu-rep --page raw --csv > gpurun_out/${R}_columns_raw.csv 2>/dev/null
# fp32 3xTF32 DCN (C4 fp32)
ncu --set full --clock-control none -k regex:"dcn_fwd" -c 1 -o gpurun_out/${R}_f32 \
    python tools/probe_dcn.py yolact_r101_c4_v2_f32 3xtf32 > /dev/null 2>&1
ncu -i gpurun_out/${R}_f32.ncu-rep --page raw --csv > gpurun_out/${R}_f32_raw.csv 2>/dev/null
echo done
