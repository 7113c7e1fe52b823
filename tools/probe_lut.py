"""the regular-conv offset-branch baseline and a per-shape latency table.

  python tools/probe_lut.py [--batch 16] [--out profiles/rNN_lut.json]

For every DCN layer shape of the YOLACT++ interval-3 stack (configs.stack_layers, at the given
per-GPU batch) and the single-layer configs C3/C4/C5 it times, on one GPU with CUDA-graph
replay and inputs resident:
  * lightweight: the paper's offset branch, defcon_offset_dw_conv;
  * regular:     the offset field as a REGULAR 3x3 conv Cin -> 3K^2 (padded to 32 channels),
                 run as a zero-offset, mask-free deformable conv on the same fused tensor-core
                 kernel (zero offsets make Eq.2 a regular conv, pinned by oracle test P1);
  * dcn:         the fused DCN layer itself (defcon_dcn_forward).
Eq.9 says the lightweight branch needs 1/6 of the regular branch's MACs (83.3 % saving
for k = 3); the table shows what that buys in microseconds on B200, where the regular conv is a
dense contraction for the tensor cores and the depthwise conv is not.  The per-shape
microseconds are the t(w_n) latency table the interval search of Eq.6 consumes.
"""
import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
from defcon_workloads import configs  # noqa: E402
import paper_conf_ipps_jayaweeralwrk24_b200 as d  # noqa: E402
from probe_stack import graph_us, make_layer  # noqa: E402

OC_PAD = 32   # 3 * K^2 = 27 offset + mask channels, padded to the kernel's 32-channel tile


def regular_branch(c, L, dev):
    """The offset field as a regular 3x3 conv: zero offsets, no mask, Cout = 27 -> 32."""
    zoff = torch.zeros_like(L["off"])
    wr = (torch.randn(OC_PAD, c.K, c.K, c.Cin, device=dev) * (2.0 / (c.Cin * c.K * c.K)) ** 0.5).to(torch.bfloat16)
    br = torch.zeros(OC_PAD, device=dev)
    yr = torch.empty((c.N, c.Ho, c.Wo, OC_PAD), device=dev, dtype=torch.bfloat16)
    ws = torch.zeros(max(16, d.defcon_dcn_workspace_size(c.N, c.H, c.W, c.Cin, OC_PAD, c.K, c.K, c.stride, c.pad,
                                                         c.dil)), dtype=torch.uint8, device=dev)
    return lambda: d.defcon_dcn_forward(L["x"], zoff, None, wr, br, stride=c.stride, pad=c.pad, dil=c.dil, y=yr,
                                        workspace=ws)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--batch", type=int, default=16)
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    dev = torch.device("cuda")
    d.load_library()
    shapes = {}
    for c in configs.stack_layers(args.batch) + [configs.C3, configs.C4, configs.C5]:
        key = (c.N, c.H, c.W, c.Cin, c.Cout, c.stride)
        if key not in shapes:
            shapes[key] = c
    rows = []
    for c in shapes.values():
        L = make_layer(c, dev)
        P = L["P"]
        light = lambda: d.defcon_offset_dw_conv(L["x"], P["dw_w"], P["dw_scale"], P["dw_shift"], P["pw_w"],
                                                P["pw_b"], K=c.K, stride=c.stride, pad=c.pad, dil=c.dil,
                                                offset=L["off"], mask=L["msk"], workspace=L["tws"])
        light()
        dcn = lambda: d.defcon_dcn_forward(L["x"], L["off"], L["msk"], L["w"], L["b"], stride=c.stride,
                                           pad=c.pad, dil=c.dil, y=L["y"], workspace=L["ws"])
        us_light, us_reg, us_dcn = graph_us(light), graph_us(regular_branch(c, L, dev)), graph_us(dcn)
        macs_light = configs.offset_branch_macs(c)
        macs_reg = c.M * c.K * c.K * c.Cin * 3 * c.K * c.K
        rows.append({"layer": c.name, "shape": f"N{c.N} {c.H}x{c.W}x{c.Cin}->{c.Ho}x{c.Wo} s{c.stride}",
                     "us_lightweight_branch": round(us_light, 2), "us_regular_branch": round(us_reg, 2),
                     "us_dcn": round(us_dcn, 2), "mac_ratio_light_over_regular": round(macs_light / macs_reg, 4),
                     "time_ratio_light_over_regular": round(us_light / us_reg, 3)})
        print(json.dumps(rows[-1]), flush=True)
    if args.out:
        with open(args.out, "w") as f:
            json.dump({"batch": args.batch, "eq9_mac_saving_k3": configs.lightweight_mac_saving(3), "rows": rows}, f,
                      indent=1)


if __name__ == "__main__":
    main()
