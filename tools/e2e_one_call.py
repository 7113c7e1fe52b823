import os, sys, torch
sys.path.insert(0, os.getcwd())
from defcon_workloads import configs, inputs
import paper_conf_ipps_jayaweeralwrk24_b200 as d
os.environ["DEFCON_HOST_CHUNKS"] = "1"
c = configs.C4; dev = torch.device("cuda"); d.load_library()
x = inputs.gen_x(c); w, b = inputs.gen_weight(c)
P = {k: torch.from_numpy(v).to(dev) for k, v in inputs.gen_offset_branch(c).items()}
wd, bd = torch.from_numpy(w).to(dev, torch.bfloat16), torch.from_numpy(b).to(dev)
xh = torch.from_numpy(x).to(torch.bfloat16).pin_memory()
yh = torch.empty((c.N, c.Ho, c.Wo, c.Cout), dtype=torch.bfloat16).pin_memory()
ws = torch.empty(d.defcon_layer_workspace_size(c.N, c.H, c.W, c.Cin, c.Cout), dtype=torch.uint8, device=dev)
for _ in range(4): d.defcon_layer_forward_host(xh, P, wd, bd, yh, ws)
torch.cuda.synchronize()
