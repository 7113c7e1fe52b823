"""Build dev-probe variants of libdefcon.so (extra -D flags) into tools/bin/ for A/B timing.

  python tools/build_variants.py name=-DFLAG[,-DFLAG2] ...
Each variant is loaded by setting DEFCON_LIB=tools/bin/libdefcon_<name>.so.
"""
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_ipps_jayaweeralwrk24_b200 import build as B  # noqa: E402


def one(spec):
    name, _, flags = spec.partition("=")
    out = os.path.join(ROOT, "tools", "bin", f"libdefcon_{name}.so")
    os.makedirs(os.path.dirname(out), exist_ok=True)
    cmd = ["/usr/local/cuda/bin/nvcc", *B.NVCC_FLAGS, *[f for f in flags.split(",") if f], "-I", B.INCLUDE,
           "-o", out, *B.sources(), "-lcudart"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode:
        print(r.stderr[-3000:])
        raise SystemExit(f"variant {name} failed")
    return name


if __name__ == "__main__":
    with ThreadPoolExecutor(4) as ex:
        for n in ex.map(one, sys.argv[1:]):
            print("built", n)
