"""Per-task timing trace of the prev-row kernel (LDDP_TRACE): task start (flags satisfied) and
end stamps per (band, block).  Development tool.

    python tools/trace_prevrow.py --rows 4096 --cols 32768
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
    ap.add_argument("--rows", type=int, default=4096)
    ap.add_argument("--cols", type=int, default=32768)
    args = ap.parse_args()
    from paper_conf_ipps_kumark15_b200 import inputs, lddp
    dev = torch.device("cuda", 0)
    c = torch.from_numpy(inputs.gen_costs(0, args.rows, args.cols)).to(dev)
    plan = lddp.Plan("minpath3", "prev_row", args.rows, args.cols, lddp.OUT_SCORE | lddp.OUT_LAST_ROW)
    info = json.loads(plan.info)
    nb, nbands = info["blocks"], info["bands"]
    s = torch.zeros(1, dtype=torch.int32, device=dev)
    lr = torch.zeros(args.cols, dtype=torch.int32, device=dev)
    plan.fill(grid=c, score=s, last_row=lr)
    torch.cuda.synchronize()
    buf = torch.zeros(nbands * nb * 2, dtype=torch.int64, device=dev)
    os.environ["LDDP_TRACE"] = f"{buf.data_ptr()}:{nb}"
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    plan.fill(grid=c, score=s, last_row=lr)
    e1.record()
    torch.cuda.synchronize()
    del os.environ["LDDP_TRACE"]
    tr = buf.cpu().numpy().reshape(nbands, nb, 2).astype(np.float64)
    tr -= tr[tr > 0].min()
    dur = tr[:, :, 1] - tr[:, :, 0]
    # latency: task start minus the latest end of its three band-(b-1) neighbours
    lat = []
    for b in range(1, nbands):
        for J in range(nb):
            dep = max(tr[b - 1, max(J - 1, 0), 1], tr[b - 1, J, 1], tr[b - 1, min(J + 1, nb - 1), 1])
            lat.append(tr[b, J, 0] - dep)
    lat = np.array(lat)
    band_end = tr[:, :, 1].max(axis=1)
    print(json.dumps({"ms": e0.elapsed_time(e1), "bands": nbands, "blocks": nb,
                      "task_us_median": float(np.median(dur)) / 1e3, "task_us_p90": float(np.percentile(dur, 90)) / 1e3,
                      "start_after_deps_us_median": float(np.median(lat)) / 1e3,
                      "start_after_deps_us_p90": float(np.percentile(lat, 90)) / 1e3,
                      "band_period_us": float(np.median(np.diff(band_end))) / 1e3}, indent=1))


if __name__ == "__main__":
    main()
