"""Device time of TABLE fills (LCS / Levenshtein / DTW n x n, the traceback inputs) per
LDDP_WF_VARIANT, CUDA events, parity of the score vs the SCORE-only plan.  Development tool.

    python tools/table_time.py --n 8192 --variant 0 2
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
    ap.add_argument("--n", type=int, default=8192)
    ap.add_argument("--variant", type=int, nargs="+", default=[0])
    ap.add_argument("--func", nargs="+", default=["lcs", "levenshtein", "dtw"])
    args = ap.parse_args()
    from paper_conf_ipps_kumark15_b200 import inputs, lddp
    dev = torch.device("cuda", 0)
    n = args.n
    for func in args.func:
        if func == "dtw":
            x, y = inputs.gen_walks(0, n, n)
            a, b = torch.from_numpy(x).to(dev), torch.from_numpy(y).to(dev)
            dt = torch.float32
        else:
            x, y = inputs.gen_strings(0, n, n)
            a, b = torch.from_numpy(x).to(dev), torch.from_numpy(y).to(dev)
            dt = torch.int32
        ref = torch.zeros(1, dtype=dt, device=dev)
        p0 = lddp.Plan(func, "anti_diagonal", n, n, lddp.OUT_SCORE)
        p0.fill(a=a, b=b, score=ref)
        s0, e0 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s0.record()
        for _ in range(5):
            p0.fill(a=a, b=b, score=ref)
        e0.record()
        torch.cuda.synchronize()
        print(json.dumps({"func": func, "n": n, "score_only_ms": round(s0.elapsed_time(e0) / 5, 3),
                          "kernel": json.loads(p0.info)["kernel"]}), flush=True)
        for v in args.variant:
            os.environ["LDDP_WF_VARIANT"] = str(v)
            tab = torch.zeros((n, n), dtype=dt, device=dev)
            sc = torch.zeros(1, dtype=dt, device=dev)
            plan = lddp.Plan(func, "anti_diagonal", n, n, lddp.OUT_SCORE | lddp.OUT_TABLE)
            for _ in range(2):
                plan.fill(a=a, b=b, score=sc, table=tab)
            plan.check()
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            for _ in range(5):
                plan.fill(a=a, b=b, score=sc, table=tab)
            e.record()
            torch.cuda.synchronize()
            ms = s.elapsed_time(e) / 5
            print(json.dumps({"func": func, "n": n, "variant": v, "ms": round(ms, 3),
                              "gcups": round(n * n / ms / 1e6, 1), "score_match": bool((sc == ref).item()),
                              "plan": json.loads(plan.info)}), flush=True)
            del tab
        os.environ.pop("LDDP_WF_VARIANT", None)


if __name__ == "__main__":
    main()
