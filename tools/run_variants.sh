for v in base same nomath samenomath st2 st4; do
  echo "== $v"; DEFCON_LIB=tools/bin/libdefcon_$v.so timeout 120 python tools/probe_dcn.py yolact_r101_c3_v2,yolact_r101_c4_v2,yolact_r101_c5_v2 ldg 2>&1 | tail -3
done
