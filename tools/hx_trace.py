"""clock64 trace of one CTA of the hierarchical-exchange prev-row kernel (LDDP_TRACE): per warp,
cycles per inner band of rows and per band including the exchange; optional LDDP_DEBUG timing
switches (1 = no outer L2 waits, 2 = no inner barrier, wrong results).  Development tool.

    python tools/hx_trace.py --cta 70 --debug 0 1 2 3

Needs a trace build: make -C paper_conf_ipps_kumark15_b200 -B EXTRA=-DLDDP_HX_TRACE (the per-band
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
    ap.add_argument("--func", default="minpath3")
    ap.add_argument("--cta", type=int, nargs="+", default=[70])
    ap.add_argument("--debug", type=int, nargs="+", default=[0])
    ap.add_argument("--hbi", type=int, default=16)
    args = ap.parse_args()
    from paper_conf_ipps_kumark15_b200 import lddp
    dev = torch.device("cuda", 0)
    H, W = args.H, args.W
    g = torch.randint(0, 1024, (H, W), dtype=torch.int32, device=dev)
    score = torch.zeros(1, dtype=torch.int32, device=dev)
    lr = torch.zeros(W, dtype=torch.int32, device=dev)
    buf = torch.zeros(2 * 4 * 4096, dtype=torch.int64, device=dev)
    plan = lddp.Plan(args.func, "prev_row", H, W, lddp.OUT_SCORE | lddp.OUT_LAST_ROW, param_c=1)
    plan.fill(grid=g, score=score, last_row=lr)
    torch.cuda.synchronize()
    nb = (H + args.hbi - 1) // args.hbi
    for dbg in args.debug:
        os.environ["LDDP_DEBUG"] = str(dbg)
        for cta in args.cta:
            buf.zero_()
            os.environ["LDDP_TRACE"] = f"{buf.data_ptr()}:{cta}"
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            plan.fill(grid=g, score=score, last_row=lr)
            e.record()
            torch.cuda.synchronize()
            del os.environ["LDDP_TRACE"]
            t = buf.cpu().numpy().reshape(-1, 4, 2).astype(np.float64)[:nb]
            out = {"debug": dbg, "cta": cta, "ms": round(s.elapsed_time(e), 4), "plan": json.loads(plan.info)["kernel"]}
            for w in range(4):
                loop = t[1:-1, w, 0] / args.hbi
                tot = t[1:-1, w, 1] / args.hbi
                out[f"w{w}"] = {"loop_cyc_row_p50": round(float(np.median(loop)), 1),
                                "tot_cyc_row_p50": round(float(np.median(tot)), 1),
                                "tot_cyc_row_mean": round(float(np.mean(tot)), 1),
                                "wait_p10_50_90_99": [round(float(np.percentile(t[1:-1, w, 1] - t[1:-1, w, 0], q))) for q in (10, 50, 90, 99)]}
            print(json.dumps(out), flush=True)
        os.environ.pop("LDDP_DEBUG", None)


if __name__ == "__main__":
    main()
