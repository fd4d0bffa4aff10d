"""One fill of each kernel that the bench line does not time, for ncu captures (development /
measurement tool): LCS 8192² TABLE fills on the adiag staging-tile kernel and on the wavefront
kernel, the traceback of that table, the claimed-task prev-row fallback (W % 4 != 0), the Vertical twin (transpose + prev-row),
the mInverted-L twin (mirrored inverted-L), a batched FS fill (4 × 4096²) and a prev-row TABLE
fill on prevrow_cb (LDDP_HX_VARIANT=-1; the bench's prev-row lines run prevrow_hx).

    ncu --set full -k regex:wavefront -c 1 python tools/prof_extra.py
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    from paper_conf_ipps_kumark15_b200 import inputs, lddp
    dev = torch.device("cuda", 0)
    n = 8192
    a, b = inputs.gen_strings(0, n, n)
    ta, tb = torch.from_numpy(a).to(dev), torch.from_numpy(b).to(dev)
    tab = torch.zeros((n, n), dtype=torch.int32, device=dev)
    sc = torch.zeros(1, dtype=torch.int32, device=dev)
    plan = lddp.Plan("lcs", "anti_diagonal", n, n, lddp.OUT_SCORE | lddp.OUT_TABLE)   # adiag, TABLE tile
    plan.fill(a=ta, b=tb, score=sc, table=tab)
    plan.check()
    os.environ["LDDP_KERNEL"] = "wavefront"   # the generic wavefront kernel on the same TABLE fill
    pw = lddp.Plan("lcs", "anti_diagonal", n, n, lddp.OUT_SCORE | lddp.OUT_TABLE)
    del os.environ["LDDP_KERNEL"]
    pw.fill(a=ta, b=tb, score=sc, table=tab)
    pw.check()
    pi, pj = plan.traceback(ta, tb, tab)
    torch.cuda.synchronize()
    del tab
    g = torch.from_numpy(inputs.gen_costs(1, n, n - 2)).to(dev)            # W % 4 != 0: fallback kernel
    lr = torch.zeros(n - 2, dtype=torch.int32, device=dev)
    p2 = lddp.Plan("minpath3", "prev_row", n, n - 2, lddp.OUT_SCORE | lddp.OUT_LAST_ROW)
    p2.fill(grid=g, score=sc, last_row=lr)
    p2.check()
    gi = torch.from_numpy(inputs.gen_init(2, n, n)).to(dev)
    lc = torch.zeros(n, dtype=torch.int32, device=dev)
    p3 = lddp.Plan("min2plus_v", "vertical", n, n, lddp.OUT_SCORE | lddp.OUT_LAST_COL)
    p3.fill(grid=gi, score=sc, last_col=lc)
    p3.check()
    lr2 = torch.zeros(n, dtype=torch.int32, device=dev)
    p4 = lddp.Plan("antidiag_maxplus", "minverted_l", n, n, lddp.OUT_LAST_ROW | lddp.OUT_LAST_COL)
    p4.fill(grid=gi, last_row=lr2, last_col=lc)
    p4.check()
    B, m = 4, 4096
    imgs = torch.from_numpy(np.concatenate([inputs.gen_image(k, m, m, "ramp") for k in range(B)])).to(dev)
    out = torch.zeros_like(imgs)
    p5 = lddp.Plan("fs", "knight_move", m, m, lddp.OUT_TABLE, batch=B)
    p5.fill(grid=imgs, table=out)
    p5.check()
    del imgs, out
    gt = torch.from_numpy(inputs.gen_costs(3, n, n)).to(dev)
    tt = torch.zeros((n, n), dtype=torch.int32, device=dev)
    os.environ["LDDP_HX_VARIANT"] = "-1"   # prevrow_cb (the multi-GPU / unaligned-TABLE kernel)
    p6 = lddp.Plan("minpath3", "prev_row", n, n, lddp.OUT_SCORE | lddp.OUT_TABLE)
    del os.environ["LDDP_HX_VARIANT"]
    p6.fill(grid=gt, score=sc, table=tt)
    p6.check()
    torch.cuda.synchronize()
    print("ok", int(sc.item()))


if __name__ == "__main__":
    main()
