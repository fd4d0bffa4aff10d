"""Sweep anti-diagonal kernel geometries (R, E, W) on a config (one input upload, one plan per
setting), device-timed like bench.py, parity-checked against the oracle's bench refs.
Development tool, not the bench contract.

    python tools/ad_sweep.py --cfg C5 --geoms 6,2,4 6,1,4 4,1,4
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
    ap.add_argument("--cfg", default="C5")
    ap.add_argument("--geoms", nargs="+", default=["6,2,4"])
    ap.add_argument("--reps", type=int, default=5)
    args = ap.parse_args()
    from paper_conf_ipps_kumark15_b200 import lddp
    dev = torch.device("cuda", 0)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    cfg = CONFIGS[args.cfg]
    pb = None
    for g in args.geoms:
        vals = [int(v) for v in g.split(",")]
        R, E, W = vals[:3]
        S = vals[3] if len(vals) > 3 else 0
        os.environ["LDDP_AD_R"], os.environ["LDDP_AD_E"], os.environ["LDDP_AD_W"] = str(R), str(E), str(W)
        os.environ["LDDP_AD_S"] = str(S)
        if pb is None:
            pb = bench.build_problem(args.cfg, dev, lddp, 1, 0)
        else:
            pb["plan"] = lddp.Plan(cfg["func"], cfg["category"], cfg["rows"], cfg["cols"], pb["outs"], device=0)
        if "score" in pb["t"]:
            pb["t"]["score"].fill_(-1)
        ms, per, _, _ = bench.time_device(pb, lddp, args.reps, 3, dev, 1, flush)
        par = bench.check_result(args.cfg, pb)
        cells = cfg["rows"] * cfg["cols"]
        print(json.dumps({"cfg": args.cfg, "geom": g, "ms": round(ms, 4), "min": round(min(per), 4),
                          "gcups": round(cells / ms / 1e6, 1), "parity": par.get("match"),
                          "plan": json.loads(pb["plan"].info)}), flush=True)


if __name__ == "__main__":
    main()
