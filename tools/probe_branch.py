"""Time the lightweight offset branch (defcon_offset_dw_conv) alone, graph-replayed, per config.

  python tools/probe_branch.py [config,...]
Prints one JSON line per config for the loaded library ("path" = PROBE_PATH, default
"onepass"); the two-launch path (dw kernel + 1x1 kernel through an HBM intermediate) is timed
with a dev build: python tools/build_variants.py two_pass=-DDEFCON_DEV_TWO_PASS, then
DEFCON_LIB=tools/bin/libdefcon_two_pass.so PROBE_PATH=two_pass python tools/probe_branch.py
"""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from defcon_workloads import configs, inputs  # noqa: E402
import paper_conf_ipps_jayaweeralwrk24_b200 as d  # noqa: E402


def time_branch(c, reps=200):
    dev = torch.device("cuda")
    x = torch.from_numpy(inputs.gen_x(c)).to(dev, torch.bfloat16 if c.dtype == "bf16" else torch.float32)
    P = {k: torch.from_numpy(v).to(dev) for k, v in inputs.gen_offset_branch(c).items()}
    KK = c.K * c.K
    off = torch.empty((c.N, c.Ho, c.Wo, c.G, KK, 2), device=dev)
    msk = torch.empty((c.N, c.Ho, c.Wo, c.G, KK), device=dev) if c.modulated else None
    tws = torch.empty(d.defcon_offset_workspace_size(c.N, c.H, c.W, c.Cin, c.K, c.stride, c.pad, c.dil, c.G),
                      dtype=torch.uint8, device=dev)
    fn = lambda: d.defcon_offset_dw_conv(x, P["dw_w"], P["dw_scale"], P["dw_shift"], P["pw_w"], P["pw_b"],
                                         K=c.K, stride=c.stride, pad=c.pad, dil=c.dil, offset_groups=c.G,
                                         with_mask=c.modulated, offset=off, mask=msk, workspace=tws)
    for _ in range(5):
        fn()
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    with torch.cuda.graph(g, stream=s):
        for _ in range(10):
            fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps // 10):
        g.replay()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) * 1e3 / reps


if __name__ == "__main__":
    names = sys.argv[1].split(",") if len(sys.argv) > 1 else ["yolact_r101_c3_v2", "yolact_r101_c4_v2",
                                                             "yolact_r101_c4_v2_g4", "yolact_r101_c5_v2"]
    d.load_library()
    for n in names:
        c = configs.SINGLE_LAYER[n] if n in configs.SINGLE_LAYER else {l.name: l for l in configs.stack_layers(64)}[n]
        us = time_branch(c)
        byt = configs.offset_branch_compulsory_bytes(c)
        print(json.dumps({"config": n, "path": os.environ.get("PROBE_PATH", "onepass"), "us": round(us, 2),
                          "GB/s(compulsory)": round(byt / (us * 1e-6) / 1e9, 1)}))
