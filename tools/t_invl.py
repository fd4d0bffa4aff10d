"""Development: one inverted-L fill (H x W) against the oracle."""
import sys
import torch
sys.path.insert(0, ".")
from paper_conf_ipps_kumark15_b200 import lddp, inputs
import oracle
H, W = int(sys.argv[1]), int(sys.argv[2])
cat = sys.argv[3] if len(sys.argv) > 3 else "inverted_l"
func = "diagmaxplus" if cat == "inverted_l" else "antidiag_maxplus"
g = inputs.gen_init(1, H, W)
t = torch.from_numpy(g).cuda()
lr = torch.zeros(W, dtype=torch.int32, device="cuda")
lc = torch.zeros(H, dtype=torch.int32, device="cuda")
p = lddp.Plan(func, cat, H, W, lddp.OUT_LAST_ROW | lddp.OUT_LAST_COL)
p.fill(grid=t, last_row=lr, last_col=lc)
p.check()
r = (oracle.diagmaxplus if func == "diagmaxplus" else oracle.antidiag_maxplus)(g, 1)
print("ok", H, W, cat, bool((lr.cpu().numpy() == r.last_row).all()), bool((lc.cpu().numpy() == r.last_col).all()))
