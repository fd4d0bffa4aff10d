"""Sweep the prev-row column-block kernel geometry on C4 (one grid upload, one plan per
setting), device-timed like bench.py, parity-checked against the oracle's bench refs.
Development tool, not the bench contract.

    python tools/cb_sweep.py --variant 0 1 2 3 4 --warps 1 2 4 --reps 5
"""
import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
import bench  # noqa: E402
from configs import CONFIGS  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--cfg", default="C4")
    ap.add_argument("--variant", type=int, nargs="*", default=[0])
    ap.add_argument("--warps", type=int, nargs="*", default=[2])
    ap.add_argument("--reps", type=int, default=5)
    args = ap.parse_args()
    from paper_conf_ipps_kumark15_b200 import lddp
    dev = torch.device("cuda", 0)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    cfg = CONFIGS[args.cfg]
    pb = None
    for var in args.variant:
        for nw in args.warps:
            os.environ["LDDP_CB_VARIANT"] = str(var)
            os.environ["LDDP_CB_WARPS"] = str(nw)
            if pb is None:
                pb = bench.build_problem(args.cfg, dev, lddp, 1, 0)
            else:
                pb["plan"] = lddp.Plan(cfg["func"], cfg["category"], cfg["rows"], cfg["cols"], pb["outs"],
                                       device=0)
            for k in ("score", "last_row"):
                if k in pb["t"]:
                    pb["t"][k].fill_(-1)
            ms, per, _, _ = bench.time_device(pb, lddp, args.reps, 3, dev, 1, flush)
            par = bench.check_result(args.cfg, pb)
            cells = cfg["rows"] * cfg["cols"]
            gbs = cells * 4 / ms / 1e6
            print(json.dumps({"cfg": args.cfg, "variant": var, "warps": nw, "ms": round(ms, 4),
                              "min": round(min(per), 4), "gcups": round(cells / ms / 1e6, 1),
                              "GBps": round(gbs, 1), "parity": par.get("match"),
                              "plan": json.loads(pb["plan"].info)}), flush=True)


if __name__ == "__main__":
    main()
