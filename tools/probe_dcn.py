"""Time the fused DCN kernel alone (graph-replayed launches) per config and sampler.

  python tools/probe_dcn.py [config[:N],...] [ldg,tex]
Prints one JSON line per (config, sampler): microseconds per launch (incl. the texture
staging pass for the TEX sampler) and contraction TFLOP/s.
"""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from defcon_workloads import configs, inputs  # noqa: E402
import paper_conf_ipps_jayaweeralwrk24_b200 as d  # noqa: E402


BOUND = int(os.environ.get("PROBE_BOUND", "0"))   # bounded deformation P (0 = unbounded)
OFF16 = os.environ.get("PROBE_OFF16", "0") == "1"  # tex2D++: binary16 offsets / mask


def time_cfg(c, sampler, reps=200):
    """sampler: ldg / tex / hybrid, or (fp32 configs) the fp32 mode simt / 3xtf32."""
    fp32_mode = sampler if sampler in ("simt", "3xtf32") else "simt"
    sampler = "ldg" if sampler in ("simt", "3xtf32") else sampler
    dev = torch.device("cuda")
    L = inputs.gen_layer(c)
    dt = torch.bfloat16 if c.dtype == "bf16" else torch.float32
    x = torch.from_numpy(L["x"]).to(dev, dt)
    odt = torch.float16 if OFF16 else torch.float32
    off = torch.from_numpy(L["offset"]).to(dev, odt)
    msk = torch.from_numpy(L["mask"]).to(dev, odt) if L["mask"] is not None else None
    w = torch.from_numpy(L["weight"]).to(dev, dt)
    b = torch.from_numpy(L["bias"]).to(dev)
    y = torch.empty((c.N, c.Ho, c.Wo, c.Cout), device=dev, dtype=dt)
    ws = torch.zeros(max(16, d.defcon_dcn_workspace_size(c.N, c.H, c.W, c.Cin, c.Cout, c.K, c.K,
                                                         c.stride, c.pad, c.dil, c.G, dt, sampler,
                                                         fp32_mode)),
                     dtype=torch.uint8, device=dev)
    plan = d.TexPlan(c.N, c.H, c.W, c.Cin, dt) if sampler in ("tex", "hybrid") else None
    fn = lambda: d.defcon_dcn_forward(x, off, msk, w, b, stride=c.stride, pad=c.pad, dil=c.dil,
                                      offset_groups=c.G, y=y, workspace=ws, sampler=sampler,
                                      tex_plan=plan, fp32_mode=fp32_mode, bound=BOUND)
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
    us = e0.elapsed_time(e1) * 1e3 / reps
    return us, configs.contraction_flops(c) / (us * 1e-6) / 1e12


if __name__ == "__main__":
    names = sys.argv[1].split(",") if len(sys.argv) > 1 else ["yolact_r101_c4_v2"]
    samplers = sys.argv[2].split(",") if len(sys.argv) > 2 else ["ldg", "tex", "hybrid"]
    d.load_library()
    for n in names:
        if ":" in n:          # name:N override, e.g. yolact_r101_c4_v2:8
            base, nn = n.split(":")
            c = configs.SINGLE_LAYER[base].replace(N=int(nn))
        else:
            c = configs.SINGLE_LAYER[n]
        for smp in samplers:
            us, tf = time_cfg(c, smp)
            print(json.dumps({"config": n, "sampler": smp, "us": round(us, 2), "tflops": round(tf, 1)}))
