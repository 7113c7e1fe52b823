"""Sampling stage on its own: defcon_deform_columns writes the bf16
deformable columns to HBM.  Reports us, HBM GB/s (column write + compulsory reads), the
fraction of measured HBM bandwidth, and sampled elements/clk/SM; plus the unfused two-step
baseline (columns + cuBLAS GEMM via torch.matmul) against the fused kernel.

  python tools/probe_sampler.py [config,...]
"""
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from defcon_workloads import configs, inputs  # noqa: E402
import paper_conf_ipps_jayaweeralwrk24_b200 as d  # noqa: E402


def graph_time(fn, reps=100):
    for _ in range(3):
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
    names = sys.argv[1].split(",") if len(sys.argv) > 1 else ["yolact_r101_c5_v2", "yolact_r101_c4_v2",
                                                             "yolact_r101_c3_v2"]
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    d.load_library()
    dev = torch.device("cuda")
    nsm = torch.cuda.get_device_properties(0).multi_processor_count
    for n in names:
        c = configs.SINGLE_LAYER[n]
        L = inputs.gen_layer(c)
        x = torch.from_numpy(L["x"]).to(dev, torch.bfloat16)
        off = torch.from_numpy(L["offset"]).to(dev)
        msk = torch.from_numpy(L["mask"]).to(dev)
        w = torch.from_numpy(L["weight"]).to(dev, torch.bfloat16)
        b = torch.from_numpy(L["bias"]).to(dev)
        KK = c.K * c.K
        cols = torch.empty((c.M, KK * c.Cin), device=dev, dtype=torch.bfloat16)
        y2 = torch.empty((c.M, c.Cout), device=dev, dtype=torch.bfloat16)
        wm = w.reshape(c.Cout, -1).t()
        t_cols = graph_time(lambda: d.defcon_deform_columns(x, off, msk, K=c.K, columns=cols))
        t_two = graph_time(lambda: (d.defcon_deform_columns(x, off, msk, K=c.K, columns=cols),
                                    torch.addmm(b.to(torch.bfloat16), cols, wm, out=y2)))
        ws = torch.zeros(d.defcon_dcn_workspace_size(c.N, c.H, c.W, c.Cin, c.Cout, c.K, c.K), dtype=torch.uint8,
                         device=dev)
        y = torch.empty((c.N, c.Ho, c.Wo, c.Cout), device=dev, dtype=torch.bfloat16)
        t_fused = graph_time(lambda: d.defcon_dcn_forward(x, off, msk, w, b, y=y, workspace=ws))
        col_bytes = c.M * KK * c.Cin * 2
        rd = c.N * c.H * c.W * c.Cin * 2 + c.M * KK * 3 * 4
        gbs = (col_bytes + rd) / (t_cols * 1e-6) / 1e9
        clk = peaks.get("sm_max_mhz", 1965.0) * 1e6
        print(json.dumps({"config": n, "columns_us": round(t_cols, 2), "columns_MB": round(col_bytes / 1e6, 1),
                          "hbm_GBps": round(gbs, 1), "hbm_frac": round(gbs / peaks["hbm_gbs"], 3),
                          "elements_per_clk_per_sm": round(c.M * KK * c.Cin / (t_cols * 1e-6) / clk / nsm, 1),
                          "two_step_us(columns+cuBLAS)": round(t_two, 2), "fused_us": round(t_fused, 2),
                          "fused_speedup_vs_two_step": round(t_two / t_fused, 2)}))
