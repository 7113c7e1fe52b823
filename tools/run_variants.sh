#!/bin/bash
# A/B the dev-probe variants built by tools/build_variants.py (one line per variant x config).
for v in ${VARIANTS:-base same nomath samenomath nob}; do
  echo "== $v"; DEFCON_LIB=tools/bin/libdefcon_$v.so timeout 120 python tools/probe_dcn.py ${CONFIGS:-yolact_r101_c3_v2,yolact_r101_c4_v2,yolact_r101_c5_v2} ldg 2>&1 | tail -6
done
