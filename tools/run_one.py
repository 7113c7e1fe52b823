"""Run the fused DCN kernel once per call on a BASELINE config (for ncu captures)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from defcon_workloads import configs, inputs  # noqa: E402
import paper_conf_ipps_jayaweeralwrk24_b200 as d  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "yolact_r101_c4_v2"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
c = configs.SINGLE_LAYER[name]
dev = torch.device("cuda")
L = inputs.gen_layer(c)
dt = torch.bfloat16 if c.dtype == "bf16" else torch.float32
x = torch.from_numpy(L["x"]).to(dev, dt)
off = torch.from_numpy(L["offset"]).to(dev)
msk = torch.from_numpy(L["mask"]).to(dev)
w = torch.from_numpy(L["weight"]).to(dev, dt)
b = torch.from_numpy(L["bias"]).to(dev)
for _ in range(reps):
    d.defcon_dcn_forward(x, off, msk, w, b, stride=c.stride, pad=c.pad, dil=c.dil, offset_groups=c.G)
torch.cuda.synchronize()
