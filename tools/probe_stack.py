"""Config 5: the interval-3 DCN stack of YOLACT++ R101 C3-C5 (11 layers),
each layer = its lightweight offset branch + the fused DCN, global batch 64 sharded by image.

  python tools/probe_stack.py [--batches 64,32,16,8] [--out profiles/rNN_stack.json]

Work shards by image with no exchange: on g GPUs each rank runs the same
stack at batch 64/g, so the per-GPU time at batch 64/g measured here on one B200 is the
g-GPU step time (the driver's own 1/2/4/8-GPU bench runs check the weak-scaling side).
Per layer: us for branch + DCN (CUDA-graph replay, inputs resident), contraction TFLOP/s.
"""
import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from defcon_workloads import configs, inputs  # noqa: E402
import paper_conf_ipps_jayaweeralwrk24_b200 as d  # noqa: E402


def make_layer(c, dev):
    x = torch.from_numpy(inputs.gen_x(c, images=range(min(c.N, 4)))).to(dev, torch.bfloat16)
    if c.N > x.shape[0]:     # tile the generated images (timing only; values stay in range)
        x = x.repeat((c.N + x.shape[0] - 1) // x.shape[0], 1, 1, 1)[: c.N].contiguous()
    P = {k: torch.from_numpy(v).to(dev) for k, v in inputs.gen_offset_branch(c).items()}
    w, b = inputs.gen_weight(c)
    KK = c.K * c.K
    L = dict(x=x, P=P, w=torch.from_numpy(w).to(dev, torch.bfloat16), b=torch.from_numpy(b).to(dev),
             off=torch.empty((c.N, c.Ho, c.Wo, c.G, KK, 2), device=dev),
             msk=torch.empty((c.N, c.Ho, c.Wo, c.G, KK), device=dev),
             y=torch.empty((c.N, c.Ho, c.Wo, c.Cout), device=dev, dtype=torch.bfloat16),
             tws=torch.empty(d.defcon_offset_workspace_size(c.N, c.H, c.W, c.Cin, c.K, c.stride, c.pad, c.dil),
                             dtype=torch.uint8, device=dev),
             ws=torch.zeros(max(16, d.defcon_dcn_workspace_size(c.N, c.H, c.W, c.Cin, c.Cout, c.K, c.K, c.stride,
                                                                 c.pad, c.dil)), dtype=torch.uint8, device=dev))
    return L


def run_layer(c, L):
    P = L["P"]
    d.defcon_offset_dw_conv(L["x"], P["dw_w"], P["dw_scale"], P["dw_shift"], P["pw_w"], P["pw_b"], K=c.K,
                            stride=c.stride, pad=c.pad, dil=c.dil, offset=L["off"], mask=L["msk"],
                            workspace=L["tws"])
    d.defcon_dcn_forward(L["x"], L["off"], L["msk"], L["w"], L["b"], stride=c.stride, pad=c.pad, dil=c.dil,
                         y=L["y"], workspace=L["ws"])


def graph_us(fn, reps=50):
    for _ in range(3):
        fn()
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    with torch.cuda.graph(g, stream=s):
        for _ in range(5):
            fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps // 5):
        g.replay()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) * 1e3 / reps


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--batches", default="64,32,16,8")
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    dev = torch.device("cuda")
    d.load_library()
    res = {"config": "full DEFCON interval-placed DCN stack (every 3rd bottleneck in C3-C5), batch 64",
           "layers": [c.name for c in configs.stack_layers(64)], "per_gpu_batch": {}}
    t1 = None
    for B in [int(v) for v in args.batches.split(",")]:
        layers = configs.stack_layers(B)
        rows, tot_us, tot_flop = [], 0.0, 0
        for c in layers:
            L = make_layer(c, dev)
            us_all = graph_us(lambda: run_layer(c, L))
            us_dcn = graph_us(lambda: d.defcon_dcn_forward(L["x"], L["off"], L["msk"], L["w"], L["b"], stride=c.stride,
                                                           pad=c.pad, dil=c.dil, y=L["y"], workspace=L["ws"]))
            f = configs.contraction_flops(c)
            rows.append({"layer": c.name, "shape": f"{c.H}x{c.W}x{c.Cin}->{c.Ho}x{c.Wo}x{c.Cout} s{c.stride}",
                         "us_layer": round(us_all, 2), "us_dcn": round(us_dcn, 2),
                         "dcn_tflops": round(f / (us_dcn * 1e-6) / 1e12, 1)})
            tot_us += us_all
            tot_flop += f
            del L
            torch.cuda.empty_cache()
        g = 64 // B
        if t1 is None:
            t1 = tot_us
        res["per_gpu_batch"][str(B)] = {"gpus_for_global_64": g, "stack_us": round(tot_us, 1),
                                        "tflops": round(tot_flop / (tot_us * 1e-6) / 1e12, 1),
                                        "projected_speedup_vs_1gpu": round(t1 / tot_us, 2),
                                        "projected_efficiency": round(t1 / (g * tot_us), 3), "layers": rows}
        print(json.dumps({"batch": B, "gpus": g, "stack_us": round(tot_us, 1),
                          "tflops": res["per_gpu_batch"][str(B)]["tflops"]}), flush=True)
    if args.out:
        json.dump(res, open(args.out, "w"), indent=1)
    print(json.dumps(res)[:2000])
