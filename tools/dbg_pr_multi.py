"""Development: locate prev-row multi-GPU (loopback) mismatches against the oracle."""
import sys
import numpy as np
import torch
sys.path.insert(0, ".")
from paper_conf_ipps_kumark15_b200 import lddp
from paper_conf_ipps_kumark15_b200 import inputs
import oracle

H, W, P = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
dev = torch.device("cuda:0")
plan = lddp.Plan("minpath3", "prev_row", H, W, lddp.OUT_SCORE | lddp.OUT_LAST_ROW | lddp.OUT_TABLE)
print(lddp.lddp_plan_describe(plan.handle))
comms = [lddp.lddp_comm_create(plan.handle, P, r) for r in range(P)]
for r in range(P):
    lddp.lddp_comm_connect_local(comms[r], comms[r + 1] if r + 1 < P else None, comms[r - 1] if r > 0 else None)
g = inputs.gen_costs(5, H, W)
tg = torch.from_numpy(g).to(dev)
sc = torch.full((P,), -7, dtype=torch.int32, device=dev)
lr = torch.full((W,), -7, dtype=torch.int32, device=dev)
tab = torch.full((H, W), -7, dtype=torch.int32, device=dev)
wss = [torch.zeros(plan.ws_bytes, dtype=torch.uint8, device=dev) for _ in range(P)]
streams = [torch.cuda.Stream(dev) for _ in range(P)]
torch.cuda.synchronize()
for r in range(P):
    inp, out = plan.io(grid=tg, score=sc[r:r + 1], last_row=lr, table=tab)
    lddp.lddp_fill_multi(plan.handle, inp, out, wss[r].data_ptr(), comms[r], streams[r].cuda_stream)
for r in range(P):
    try:
        lddp.lddp_status_check(plan.handle, wss[r].data_ptr(), streams[r].cuda_stream)
    except Exception as e:
        print("rank", r, "status", e)
torch.cuda.synchronize()
ref = oracle.minpath3(g, table=True)
t = tab.cpu().numpy()
bad = t != ref.table
print("bad", bad.sum())
if bad.any():
    rr, cc = np.nonzero(bad)
    print("first bad row", rr.min(), "cols", np.unique(cc)[:40], "...", np.unique(cc)[-10:])
    r0 = rr.min()
    cs = np.unique(cc[rr == r0])
    print("row", r0, "cols", cs[:20], t[r0, cs[:8]], ref.table[r0, cs[:8]])
    for r in [r0, r0 + 1, r0 + 5]:
        print(r, np.unique(cc[rr == r])[:20])
