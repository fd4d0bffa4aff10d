"""Time FS fills of an H x W image for several H (fixed W): separates the per-step cost (the slope
in W) from the pipeline lag (the slope in H).  Development tool.

    python tools/fs_scan.py --W 8192 --H 32 128 512 2048 8192
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
    ap.add_argument("--W", type=int, default=8192)
    ap.add_argument("--H", type=int, nargs="+", default=[32, 128, 512, 2048, 8192])
    ap.add_argument("--reps", type=int, default=5)
    args = ap.parse_args()
    from paper_conf_ipps_kumark15_b200 import inputs, lddp
    dev = torch.device("cuda", 0)
    for H in args.H:
        img = torch.from_numpy(inputs.gen_image(0, H, args.W, "ramp")).to(dev)
        out = torch.zeros_like(img)
        plan = lddp.Plan("fs", "knight_move", H, args.W, lddp.OUT_TABLE)
        for _ in range(3):
            plan.fill(grid=img, table=out)
        torch.cuda.synchronize()
        ms = []
        for _ in range(args.reps):
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            plan.fill(grid=img, table=out)
            e.record()
            torch.cuda.synchronize()
            ms.append(s.elapsed_time(e))
        plan.check()
        t = sorted(ms)[len(ms) // 2]
        print(json.dumps({"H": H, "W": args.W, "ms": round(t, 4), "cycles_1965": round(t * 1.965e6),
                          "kernel": json.loads(plan.info)["kernel"]}), flush=True)


if __name__ == "__main__":
    main()
