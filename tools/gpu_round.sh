#!/bin/bash
# One GPU-box pass: gpu tests, per-config kernel probe, bench + ncu captures (round tag $1).
set -u
R=${1:-r02}
mkdir -p gpurun_out
python paper_conf_ipps_jayaweeralwrk24_b200/build.py > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/${R}_pytest_gpu.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${R}_smoke.txt 2>&1
timeout 600 python tools/probe_dcn.py yolact_r101_c3_v2,yolact_r101_c4_v2,yolact_r101_c4_v2_g4,yolact_r101_c5_v2 ldg,tex > gpurun_out/${R}_probe.jsonl 2>&1
timeout 1200 bash tools/capture_profiles.sh ${R}
