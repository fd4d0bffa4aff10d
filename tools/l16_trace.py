"""Per-strip trace of one lcs16 fill (LDDP_TRACE): claim time, first-data time, end time, cycles,
top-wait cycles, SM and hardware warp slot.  Development tool.
    python tools/l16_trace.py --cfg C5 [--out gpurun_out/l16_strips.npy]"""
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--cfg", default="C5")
    ap.add_argument("--out", default="gpurun_out/l16_strips.npy")
    args = ap.parse_args()
    from paper_conf_ipps_kumark15_b200 import lddp
    dev = torch.device("cuda", 0)
    pb = bench.build_problem(args.cfg, dev, lddp, 1, 0)
    info = json.loads(pb["plan"].info)
    S = info["strips"]
    buf = torch.zeros(S * 8, dtype=torch.int64, device=dev)
    stream = torch.cuda.current_stream(dev)
    bench.do_fill(pb, lddp, stream)
    torch.cuda.synchronize()
    os.environ["LDDP_TRACE"] = f"{buf.data_ptr()}:1"
    bench.do_fill(pb, lddp, stream)
    torch.cuda.synchronize()
    del os.environ["LDDP_TRACE"]
    tr = buf.cpu().numpy().reshape(S, 8)
    np.save(args.out, tr)
    t0 = tr[:, 0].min()
    first = (tr[:, 4] - t0) / 1e3
    end = (tr[:, 1] - t0) / 1e3
    sm = tr[:, 5] >> 32
    wslot = tr[:, 5] & 0xFFFFFFFF
    rate = (end - first)
    print(json.dumps({"strips": S, "end_us_max": float(end.max()), "first_us": [round(float(x), 1) for x in first[::52]],
                      "end_us": [round(float(x), 1) for x in end[::52]],
                      "busy_us_after_first": [round(float(x), 1) for x in rate[::52]],
                      "wait_frac": float(tr[:, 3].sum() / tr[:, 2].sum()),
                      "pre_cycles_per_chunk": float(tr[:, 6].mean() / (int(info["chunks"]) + 2 * int(info["extra_lag"]))),
                      "body_cycles_per_chunk": float(tr[:, 7].mean() / (int(info["chunks"]) + 2 * int(info["extra_lag"]))),
                      "sm_counts": np.bincount(np.bincount(sm)).tolist(),
                      "smsp_collisions": int(sum(len(v) - len(set(v)) for v in
                                                 [[int(w) % 4 for w, s_ in zip(wslot, sm) if s_ == k] for k in set(sm.tolist())]))}))


if __name__ == "__main__":
    main()
