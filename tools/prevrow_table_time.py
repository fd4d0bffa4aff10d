"""Device time of prev-row TABLE fills (MIN_PATH3, n x n) on prevrow_hx and prevrow_cb
(LDDP_HX_VARIANT=-1), CUDA events.  Development tool.

    python tools/prevrow_table_time.py --n 8192 32768
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
    ap.add_argument("--n", type=int, nargs="+", default=[8192])
    args = ap.parse_args()
    from paper_conf_ipps_kumark15_b200 import lddp
    dev = torch.device("cuda:0")
    for n in args.n:
        g = torch.randint(0, 1024, (n, n), dtype=torch.int32, device=dev)
        tab = torch.empty((n, n), dtype=torch.int32, device=dev)
        sc = torch.zeros(1, dtype=torch.int32, device=dev)
        ref = None
        for hx in ("2", "-1"):
            os.environ["LDDP_HX_VARIANT"] = hx
            p = lddp.Plan("minpath3", "prev_row", n, n, lddp.OUT_SCORE | lddp.OUT_TABLE)
            p.fill(grid=g, score=sc, table=tab)
            p.check()
            s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s.record()
            for _ in range(3):
                p.fill(grid=g, score=sc, table=tab)
            e.record()
            torch.cuda.synchronize()
            ms = s.elapsed_time(e) / 3
            sig = int(tab[n - 1].sum().item()) + int(sc.item())
            ref = sig if ref is None else ref
            print(json.dumps({"n": n, "kernel": json.loads(p.info)["kernel"], "ms": round(ms, 3),
                              "GB/s (read + table write)": round(8.0 * n * n / ms / 1e6, 1), "same_result": sig == ref}),
                  flush=True)
        os.environ.pop("LDDP_HX_VARIANT", None)
        del g, tab


if __name__ == "__main__":
    main()
