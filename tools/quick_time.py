"""Quick per-config / per-variant device timing (CUDA events, L2 flushed between fills) with the
bench's parity check.  Development tool, not the bench contract.

    python tools/quick_time.py C5 C2 --rows 4 8 --variant 0 1 --reps 5
"""
import argparse
import json
import os
import sys
import time

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
import bench  # noqa: E402
from configs import CONFIGS  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("configs", nargs="+")
    ap.add_argument("--rows", type=int, nargs="*", default=[0])
    ap.add_argument("--variant", type=int, nargs="*", default=[-1])
    ap.add_argument("--grid", type=int, nargs="*", default=[0])
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--env", nargs="*", default=[], help="KEY=v1,v2,... swept (outer product)")
    args = ap.parse_args()
    from paper_conf_ipps_kumark15_b200 import lddp
    dev = torch.device("cuda", 0)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    import itertools
    keys = [e.split("=")[0] for e in args.env]
    vals = [e.split("=")[1].split(",") for e in args.env]
    for combo in (itertools.product(*vals) if keys else [()]):
      for k, v in zip(keys, combo):
        os.environ[k] = v
      for name in args.configs:
        for rows in args.rows:
            for var in args.variant:
                for g in args.grid:
                    if var >= 0:
                        os.environ["LDDP_WF_VARIANT"] = str(var)
                    else:
                        os.environ.pop("LDDP_WF_VARIANT", None)
                    os.environ["LDDP_GRID_CTAS"] = str(g)
                    t0 = time.time()
                    try:
                        pb = bench.build_problem(name, dev, lddp, 1, 0, tile_rows=rows)
                        ms, per, _, _ = bench.time_device(pb, lddp, args.reps, 2, dev, 1, flush)
                        par = bench.check_result(name, pb)
                        cells = CONFIGS[name]["rows"] * CONFIGS[name]["cols"]
                        print(json.dumps({"env": dict(zip(keys, combo)), "cfg": name, "rows": rows, "variant": var, "grid": g,
                                          "ms": round(ms, 4), "min": round(min(per), 4),
                                          "gcups": round(cells / ms / 1e6, 1), "parity": par.get("match"),
                                          "plan": json.loads(pb["plan"].info)}), flush=True)
                    except Exception as e:  # keep going
                        print(json.dumps({"env": dict(zip(keys, combo)), "cfg": name, "rows": rows, "variant": var, "error": str(e)[:300]}), flush=True)
                    torch.cuda.empty_cache()
                    print(f"# {name} took {time.time() - t0:.1f}s", flush=True)


if __name__ == "__main__":
    main()
