#!/bin/bash
# A/B the offset-branch kernels of dev variants built by tools/build_variants.py.
for v in ${VARIANTS:-base lb3 lb5}; do
  echo "== $v"; DEFCON_LIB=tools/bin/libdefcon_$v.so timeout 120 python tools/probe_branch.py ${CONFIGS:-yolact_r101_c3_v2,yolact_r101_c4_v2,yolact_r101_c5_v2} 2>&1 | grep two_pass
done
