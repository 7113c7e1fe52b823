"""SURVEY 8(f) NEXT 3 (measurement side): sweep the runtime schedule knobs per layer shape and
record the fastest setting (the paper's Fig.8 point: the tiling / schedule choice moves the time).

  python tools/autotune.py [--out profiles/rNN_autotune.json]

Knobs (all read by the library at launch time):
  DCN     DEFCON_DCN_PAIR (single CTA / CTA pair), DEFCON_MAX_CTAS (persistent grid size)
  branch  DEFCON_OFFSET_IMPL (two_pass / tc / row_tc), DEFCON_PW_IMPL (tc / mma)
Times: CUDA-graph replay with warm L2 (tools/probe_dcn.py, tools/probe_branch.py).
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
from defcon_workloads import configs  # noqa: E402
import paper_conf_ipps_jayaweeralwrk24_b200 as d  # noqa: E402
from probe_branch import time_branch  # noqa: E402
from probe_dcn import time_cfg  # noqa: E402

KNOBS = ("DEFCON_DCN_PAIR", "DEFCON_MAX_CTAS", "DEFCON_OFFSET_IMPL", "DEFCON_PW_IMPL")


def with_env(env, fn):
    for k in KNOBS:
        os.environ.pop(k, None)
    os.environ.update(env)
    try:
        return fn()
    finally:
        for k in env:
            os.environ.pop(k, None)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    d.load_library()
    names = ["yolact_r101_c3_v2", "yolact_r101_c4_v2", "yolact_r101_c4_v2_g4", "yolact_r101_c5_v2"]
    dcn_space = [{}] + [{"DEFCON_DCN_PAIR": "1"}] + [{"DEFCON_MAX_CTAS": str(n)} for n in (74, 120, 144)]
    br_space = [{}, {"DEFCON_PW_IMPL": "tc"}, {"DEFCON_PW_IMPL": "mma"}, {"DEFCON_OFFSET_IMPL": "tc"},
                {"DEFCON_OFFSET_IMPL": "row_tc"}]
    out = {}
    for n in names:
        c = configs.SINGLE_LAYER[n]
        dcn = [(env, with_env(env, lambda: time_cfg(c, "ldg", reps=100)[0])) for env in dcn_space]
        br = [(env, with_env(env, lambda: time_branch(c, reps=100))) for env in br_space]
        bd, bb = min(dcn, key=lambda t: t[1]), min(br, key=lambda t: t[1])
        out[n] = {"dcn": [{"env": e, "us": round(u, 2)} for e, u in dcn],
                  "branch": [{"env": e, "us": round(u, 2)} for e, u in br],
                  "best_dcn": {"env": bd[0], "us": round(bd[1], 2)},
                  "best_branch": {"env": bb[0], "us": round(bb[1], 2)}}
        print(json.dumps({"config": n, "best_dcn": out[n]["best_dcn"], "default_dcn_us": out[n]["dcn"][0]["us"],
                          "best_branch": out[n]["best_branch"],
                          "default_branch_us": out[n]["branch"][0]["us"]}), flush=True)
    if args.out:
        with open(args.out, "w") as f:
            json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
