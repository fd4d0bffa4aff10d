"""clock64 trace of one prev-row column block (LDDP_TRACE): cycles per band of rows and per band
including the halo exchange.  Development tool.

    python tools/cb_trace.py --H 32768 --W 32768 --block 100

Needs a trace build: make -C paper_conf_ipps_kumark15_b200 -B EXTRA=-DLDDP_CB_TRACE (the per-band
trace checks are compiled out of the product build).
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--H", type=int, default=32768)
    ap.add_argument("--W", type=int, default=32768)
    ap.add_argument("--block", type=int, nargs="+", default=[100])
    args = ap.parse_args()
    from paper_conf_ipps_kumark15_b200 import lddp
    dev = torch.device("cuda", 0)
    H, W = args.H, args.W
    g = torch.randint(0, 1024, (H, W), dtype=torch.int32, device=dev)
    score = torch.zeros(1, dtype=torch.int32, device=dev)
    lr = torch.zeros(W, dtype=torch.int32, device=dev)
    buf = torch.zeros(2 * 4096, dtype=torch.int64, device=dev)
    plan = lddp.Plan("minpath3", "prev_row", H, W, lddp.OUT_SCORE | lddp.OUT_LAST_ROW)
    plan.fill(grid=g, score=score, last_row=lr)
    torch.cuda.synchronize()
    for blk in args.block:
        run(args, lddp, plan, g, score, lr, buf, blk, H)


def run(args, lddp, plan, g, score, lr, buf, blk, H):
    buf.zero_()
    os.environ["LDDP_TRACE"] = f"{buf.data_ptr()}:{blk}"
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    plan.fill(grid=g, score=score, last_row=lr)
    e.record()
    torch.cuda.synchronize()
    del os.environ["LDDP_TRACE"]
    t = buf.cpu().numpy().reshape(-1, 2).astype(np.float64)
    info = json.loads(plan.info)
    hb = {5: 32, 6: 32, 8: 32, 10: 32, 1: 32, 13: 16, 14: 16, 17: 48, 18: 48}.get(info["variant"], 64)
    nb = (H + hb - 1) // hb
    t = t[: nb]
    rows_c = t[:, 0] / hb
    tot_c = t[:, 1] / hb
    print(json.dumps({"block": blk, "ms": s.elapsed_time(e), "variant": info["variant"], "band_rows": hb,
                      "cycles_per_row_loop_median": float(np.median(rows_c[1:-1])),
                      "cycles_per_row_with_exchange_median": float(np.median(tot_c[1:-1])),
                      "first_bands_loop": [float(x) for x in rows_c[:6]],
                      "loop_pct_10_50_90_99": [float(np.percentile(t[1:-1, 0], q)) for q in (10, 50, 90, 99)],
                      "wait_pct_10_50_90_99": [float(np.percentile(t[1:-1, 1] - t[1:-1, 0], q)) for q in (10, 50, 90, 99)],
                      "total_cycles_block": float(t[:-1, 1].sum() + t[-1, 0])}))


if __name__ == "__main__":
    main()
