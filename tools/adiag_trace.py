"""Trace one anti-diagonal (adiag) fill with LDDP_TRACE: per (strip, warp) globaltimer start /
end, clock64 cycles, cycles spent waiting for top values and for ring back-pressure.  Prints
where the time goes.  Development tool.

    python tools/adiag_trace.py --cfg C5
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
import bench  # noqa: E402
from configs import CONFIGS  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--cfg", default="C5")
    args = ap.parse_args()
    from paper_conf_ipps_kumark15_b200 import lddp
    dev = torch.device("cuda", 0)
    pb = bench.build_problem(args.cfg, dev, lddp, 1, 0)
    info = json.loads(pb["plan"].info)
    S, W = info["strips"], info["warps"]
    buf = torch.zeros(S * W * 6, dtype=torch.int64, device=dev)
    stream = torch.cuda.current_stream(dev)
    bench.do_fill(pb, lddp, stream)
    torch.cuda.synchronize()
    os.environ["LDDP_TRACE"] = f"{buf.data_ptr()}:1"
    pb["plan"] = lddp.Plan(pb["cfg"]["func"], pb["cfg"]["category"], pb["cfg"]["rows"], pb["cfg"]["cols"],
                           pb["outs"], device=0)
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    bench.do_fill(pb, lddp, stream)
    e.record()
    torch.cuda.synchronize()
    del os.environ["LDDP_TRACE"]
    tr = buf.cpu().numpy().reshape(S, W, 6).astype(np.float64)
    t0 = tr[:, :, 0].min()
    start, end = tr[:, :, 0] - t0, tr[:, :, 1] - t0
    cyc, wt, wb = tr[:, :, 2], tr[:, :, 3], tr[:, :, 4]
    n = CONFIGS[args.cfg]["cols"]
    R, E = info["rows_per_lane"], info["extra_lag"]
    steps = n + 31 * E + 32 * E   # columns + lane lag + chunk slack (approx.)
    busy = cyc - wt - wb
    out = {"ms": s.elapsed_time(e), "plan": info,
           "warp_ns_mean": float((end - start).mean()), "warp_cycles_mean": float(cyc.mean()),
           "wait_top_frac": float(wt.sum() / cyc.sum()), "wait_bp_frac": float(wb.sum() / cyc.sum()),
           "busy_cycles_per_step": float(busy.mean() / steps),
           "cycles_per_step_incl_waits": float(cyc.mean() / steps),
           "start_lag_ns_per_warp": float(np.diff(start.reshape(-1)).mean()),
           "last_end_ns": float(end.max()), "first_start_ns": [float(x) for x in start.reshape(-1)[:12]],
           "strip_start_ns": [float(x) for x in start[:8, 0]],
           "end_ns_last_strip": [float(x) for x in end[-1]],
           "busy_cycles_per_step_by_warp": [float((busy[:, w]).mean() / steps) for w in range(W)],
           "wait_top_frac_by_warp": [float(wt[:, w].sum() / cyc[:, w].sum()) for w in range(W)]}
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
