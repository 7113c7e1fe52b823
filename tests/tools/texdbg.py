import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np, torch
import oracle
from defcon_workloads import configs, inputs
import paper_conf_ipps_jayaweeralwrk24_b200 as d
from test_gpu_parity import run_dcn, small, normwise
dev = torch.device("cuda")
for dist in ["zeros", "normal"]:
    for G in [1, 2]:
        c = small("g", G=G, Cin=128, Cout=64)
        L = inputs.gen_layer(c, off_dist=dist)
        if G == 2:   # identical offsets/mask for both groups -> must equal the G=1 result
            L["offset"][:, :, :, 1] = L["offset"][:, :, :, 0]
            L["mask"][:, :, :, 1] = L["mask"][:, :, :, 0]
        ref = oracle.dcn_forward(L["x"], L["offset"], L["weight"], L["bias"], mask=L["mask"], G=c.G)
        plan = d.TexPlan(c.N, c.H, c.W, c.Cin, torch.bfloat16)
        yt = run_dcn(d, dev, c, dict(L), sampler="tex", tex_plan=plan)
        yr = yt.reshape(-1, c.Cout); rr = ref.reshape(-1, c.Cout)
        err = np.abs(yr - rr).max(1)
        bad = np.where(err > 0.05 * np.abs(rr).max())[0]
        print(dist, G, "tex", normwise(yt, ref), "bad", bad[:12], yr[bad[:2], :4] if len(bad) else "")
