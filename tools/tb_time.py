"""Device time of lddp_traceback on n x n TABLE fills (CUDA events).  Development tool.

    python tools/tb_time.py --n 8192
"""
import argparse
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=8192)
    args = ap.parse_args()
    from paper_conf_ipps_kumark15_b200 import inputs, lddp
    dev = torch.device("cuda:0")
    n = args.n
    for f in ("lcs", "levenshtein", "dtw"):
        if f == "dtw":
            a, b = inputs.gen_walks(0, n, n)
            dt = torch.float32
        else:
            a, b = inputs.gen_strings(0, n, n)
            dt = torch.int32
        ta, tb = torch.from_numpy(a).to(dev), torch.from_numpy(b).to(dev)
        tab = torch.zeros((n, n), dtype=dt, device=dev)
        p = lddp.Plan(f, "anti_diagonal", n, n, lddp.OUT_TABLE)
        p.fill(a=ta, b=tb, table=tab)
        p.check()
        p.traceback(ta, tb, tab)
        s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s.record()
        pi, pj = p.traceback(ta, tb, tab)
        e.record()
        torch.cuda.synchronize()
        print(f, "n", n, "traceback ms", round(s.elapsed_time(e), 3), "path", len(pi), flush=True)


if __name__ == "__main__":
    main()
