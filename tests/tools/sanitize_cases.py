"""Small end-to-end cases for compute-sanitizer: every kernel of the hot
path once, on shapes the sanitizer finishes in seconds -- config 1 (tiny DCNv1 fp32), a reduced
C4 (bf16 tensor cores) with far-out-of-bounds offsets, stream-K at 3 and 37 CTAs and CTA pairs,
fp32 3xTF32, the TEX sampler, bounded deformation, the columns kernel, and both offset-branch
paths (one-pass; two-launch for wide rows).  Each case is checked loosely against the oracle
(the parity suite holds the tight gates).

  compute-sanitizer --tool memcheck python tests/tools/sanitize_cases.py
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402  (test infrastructure: the checker)
from defcon_workloads import configs, inputs  # noqa: E402
import paper_conf_ipps_jayaweeralwrk24_b200 as d  # noqa: E402

dev = torch.device("cuda")
T = {"f32": torch.float32, "bf16": torch.bfloat16}


def dv(a, dt):
    return None if a is None else torch.from_numpy(np.ascontiguousarray(a)).to(dev, dt)


def err(g, r):
    return float(np.max(np.abs(np.asarray(g, np.float64) - r)) / max(np.max(np.abs(r)), 1e-30))


def dcn(c, L, **kw):
    dt = T[c.dtype]
    y = d.defcon_dcn_forward(dv(L["x"], dt), dv(L["offset"], torch.float32), dv(L["mask"], torch.float32),
                             dv(L["weight"], dt), dv(L["bias"], torch.float32), stride=c.stride, pad=c.pad,
                             dil=c.dil, offset_groups=c.G, **kw)
    torch.cuda.synchronize()
    return y.float().cpu().numpy()


def check(name, c, L, tol, bound=0, **kw):
    y = dcn(c, L, bound=bound, **kw)
    off = oracle.bound_offsets(L["offset"], bound, K=c.K, dil=c.dil) if bound else L["offset"]
    ref = oracle.dcn_forward(L["x"], off, L["weight"], L["bias"], mask=L["mask"], stride=c.stride, pad=c.pad,
                             dil=c.dil, G=c.G)
    e = err(y, ref)
    print(f"{name}: {e:.2e}", flush=True)
    assert e < tol, name


def main():
    d.load_library()
    check("tiny_f32", configs.TINY, inputs.gen_layer(configs.TINY), 1e-4)
    c4 = configs.C4.replace(N=2, H=19, W=17)
    check("c4_bf16", c4, inputs.gen_layer(c4), 2e-2)
    check("c4_bf16_far", c4, inputs.gen_layer(c4, off_dist="far", x_dist="normal"), 2e-2)
    for ctas in ("3", "37"):
        os.environ["DEFCON_MAX_CTAS"] = ctas
        check(f"c4_bf16_streamk{ctas}", c4, inputs.gen_layer(c4), 2e-2)
        os.environ["DEFCON_DCN_PAIR"] = "1"
        check(f"c4_bf16_pair_streamk{ctas}", c4, inputs.gen_layer(c4), 2e-2)
        os.environ.pop("DEFCON_DCN_PAIR")
    os.environ.pop("DEFCON_MAX_CTAS")
    cf = c4.replace(dtype="f32", Cin=64, Cout=64)
    check("c4_f32_3xtf32", cf, inputs.gen_layer(cf), 1e-4, fp32_mode="3xtf32")
    check("c4_f32_simt", cf, inputs.gen_layer(cf), 1e-4)
    check("c4_bf16_bounded", c4, inputs.gen_layer(c4, off_dist="local"), 2e-2, bound=7)
    ct = c4.replace(Cin=64, Cout=64)
    plan = d.TexPlan(ct.N, ct.H, ct.W, ct.Cin, torch.bfloat16)
    check("c4_tex", ct, inputs.gen_layer(ct), 1e-2, sampler="tex", tex_plan=plan)
    plan.close()
    L = inputs.gen_layer(ct)
    cols = d.defcon_deform_columns(dv(L["x"], torch.bfloat16), dv(L["offset"], torch.float32),
                                   dv(L["mask"], torch.float32), K=3)
    torch.cuda.synchronize()
    ref = oracle.deform_columns(L["x"], L["offset"], 3, mask=L["mask"])
    print(f"columns: {err(cols.float().cpu().numpy(), ref):.2e}", flush=True)
    for cb in (c4, configs.LayerConfig("wide", N=1, Cin=16, Cout=16, H=20, W=300, config_id=100)):
        x = inputs.gen_x(cb)
        P = inputs.gen_offset_branch(cb)
        Pd = {k: dv(v, torch.float32) for k, v in P.items()}
        off, msk = d.defcon_offset_dw_conv(dv(x, torch.bfloat16), Pd["dw_w"], Pd["dw_scale"], Pd["dw_shift"],
                                           Pd["pw_w"], Pd["pw_b"], K=3)
        torch.cuda.synchronize()
        ro, _ = oracle.offset_branch(x, P["dw_w"], P["dw_scale"], P["dw_shift"], P["pw_w"], P["pw_b"], K=3)
        e = err(off.cpu().numpy(), ro)
        print(f"branch_{cb.name}: {e:.2e}", flush=True)
        assert e < 1e-4
    print("sanitize cases done")


if __name__ == "__main__":
    main()
