"""Texture-filter arithmetic probe (reading R14): how far is the hardware
bilinear filter of the TEX sampler from the 1/256-fraction model?

A K=1 DCNv1 with identity weights (Cin = Cout = 64, bias 0) makes y = bf16(A) = bf16(sample):
the tensor-core accumulation of a single term is exact.  y is compared element by element,
in bf16 ulps, with bf16(model sample) for the exact oracle and the texture model, for the
TEX and the LDG sampler.  Prints one JSON line per sampler.
"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import oracle  # noqa: E402  (test/tool infrastructure)
import paper_conf_ipps_jayaweeralwrk24_b200 as d  # noqa: E402


def bf16(a):
    return torch.from_numpy(np.asarray(a, np.float32)).to(torch.bfloat16).float().numpy().astype(np.float64)


def main():
    dev = torch.device("cuda:0")
    r = np.random.default_rng(5)
    N, H, W, C = 2, 23, 19, 64
    x = bf16(np.maximum(r.standard_normal((N, H, W, C)), 0) + 0.25 * r.standard_normal((N, H, W, C)))
    off = 1.5 * r.standard_normal((N, H, W, 1, 1, 2))
    w = np.eye(C).reshape(C, 1, 1, C)
    xd = torch.from_numpy(x).to(dev, torch.bfloat16)
    od = torch.from_numpy(off).to(dev, torch.float32)
    wd = torch.from_numpy(w).to(dev, torch.bfloat16)
    offr = od.cpu().double().numpy()                    # the fp32 offsets the GPU sees
    exact = oracle.dcn_forward(x, offr, w, None, mask=None, pad=0)
    model = oracle.dcn_forward_texq(x, offr, w, None, mask=None, pad=0, quant="round")
    plan = d.TexPlan(N, H, W, C, torch.bfloat16)
    for sampler in ("ldg", "tex"):
        y = d.defcon_dcn_forward(xd, od, None, wd, None, pad=0, sampler=sampler,
                                 tex_plan=plan if sampler == "tex" else None)
        torch.cuda.synchronize()
        y = y.float().cpu().double().numpy()
        out = {"sampler": sampler}
        for name, ref in (("exact", exact), ("model", model)):
            rb = bf16(ref)
            ulp = np.maximum(np.abs(rb), 1e-30)
            ulp = 2.0 ** (np.floor(np.log2(ulp)) - 7)
            du = np.abs(y - rb) / ulp
            big = np.abs(rb) > 1e-2
            out[name] = {"frac_eq": float(np.mean(du[big] == 0)), "frac_1ulp": float(np.mean(du[big] == 1)),
                         "frac_gt1ulp": float(np.mean(du[big] > 1)), "max_ulp": float(du[big].max()),
                         "max_abs_err_vs_unrounded": float(np.max(np.abs(y - ref))),
                         "normwise": float(np.max(np.abs(y - ref)) / np.max(np.abs(ref)))}
        print(json.dumps(out))
        if sampler == "tex" and os.environ.get("TEX_PROBE_DUMP"):
            np.savez(os.environ["TEX_PROBE_DUMP"], x=x, off=offr, y=y)
    plan.close()


if __name__ == "__main__":
    main()
