"""Time prev-row (MIN_PATH3) fills for several (H, W) shapes with the current env geometry:
per-row cost vs the number of column blocks.  Development tool.

    LDDP_DEBUG=56 python tools/cb_scan.py --shapes 32768x4096 32768x32768
"""
import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--shapes", nargs="+", default=["32768x4096", "32768x32768"])
    ap.add_argument("--reps", type=int, default=3)
    args = ap.parse_args()
    from paper_conf_ipps_kumark15_b200 import lddp
    dev = torch.device("cuda", 0)
    for sh in args.shapes:
        H, W = (int(v) for v in sh.split("x"))
        g = torch.randint(0, 1024, (H, W), dtype=torch.int32, device=dev)
        score = torch.zeros(1, dtype=torch.int32, device=dev)
        lr = torch.zeros(W, dtype=torch.int32, device=dev)
        plan = lddp.Plan("minpath3", "prev_row", H, W, lddp.OUT_SCORE | lddp.OUT_LAST_ROW)
        for _ in range(2):
            plan.fill(grid=g, score=score, last_row=lr)
        torch.cuda.synchronize()
        ms = []
        for _ in range(args.reps):
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            plan.fill(grid=g, score=score, last_row=lr)
            e.record()
            torch.cuda.synchronize()
            ms.append(s.elapsed_time(e))
        t = min(ms)
        info = json.loads(plan.info)
        print(json.dumps({"H": H, "W": W, "ms": round(t, 4), "cyc_per_row": round(t * 1.965e6 / H, 1),
                          "blocks": info["blocks"], "grid": info["grid"], "kernel": info["kernel"]}), flush=True)
        del g


if __name__ == "__main__":
    main()
