"""Loopback timing of the multi-GPU column-strip fill on ONE GPU (development / model-validation
tool for DESIGN.md §5.4): P virtual ranks in one process (lddp_comm_connect_local), each on its
own stream, all started after one event; device time from that event to the last rank's end.
Compares with the single-rank fill of the same problem: T(P) - T(1) measures the cross-rank
handoff term of the T(P) model (the ranks share one GPU's SMs, so this is an upper bound).

    python tools/multi_loopback_time.py --m 100000 --n 100000 --P 1 2 4
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
    ap.add_argument("--m", type=int, default=100000)
    ap.add_argument("--n", type=int, default=100000)
    ap.add_argument("--P", type=int, nargs="+", default=[1, 2, 4])
    ap.add_argument("--reps", type=int, default=3)
    args = ap.parse_args()
    from paper_conf_ipps_kumark15_b200 import inputs, lddp
    dev = torch.device("cuda:0")
    m, n = args.m, args.n
    a, b = inputs.gen_strings(0, m, n)
    ta, tb = torch.from_numpy(a).to(dev), torch.from_numpy(b).to(dev)
    plan = lddp.Plan("lcs", "anti_diagonal", m, n, lddp.OUT_SCORE | lddp.OUT_LAST_ROW | lddp.OUT_LAST_COL)
    for P in args.P:
        comms = [lddp.lddp_comm_create(plan.handle, P, g) for g in range(P)]
        for g in range(P):
            lddp.lddp_comm_connect_local(comms[g], comms[g + 1] if g + 1 < P else None, comms[g - 1] if g > 0 else None)
        sc = torch.zeros(1, dtype=torch.int32, device=dev)
        lr = torch.zeros(n, dtype=torch.int32, device=dev)
        lc = torch.zeros(m, dtype=torch.int32, device=dev)
        wss = [torch.zeros(plan.ws_bytes, dtype=torch.uint8, device=dev) for _ in range(P)]
        streams = [torch.cuda.Stream(dev) for _ in range(P)]
        times = []
        for rep in range(args.reps + 1):
            torch.cuda.synchronize()
            start = torch.cuda.Event(enable_timing=True)
            start.record(streams[0])
            ends = []
            for g in range(P):
                streams[g].wait_event(start)
                inp, out = plan.io(a=ta, b=tb, score=sc, last_row=lr, last_col=lc)
                lddp.lddp_fill_multi(plan.handle, inp, out, wss[g].data_ptr(), comms[g], streams[g].cuda_stream)
                e = torch.cuda.Event(enable_timing=True)
                e.record(streams[g])
                ends.append(e)
            torch.cuda.synchronize()
            if rep > 0:
                times.append(max(start.elapsed_time(e) for e in ends))
        for g in range(P):
            lddp.lddp_status_check(plan.handle, wss[g].data_ptr(), streams[g].cuda_stream)
        print(json.dumps({"P": P, "m": m, "n": n, "ms": round(float(np.median(times)), 3), "score": int(sc.item())}),
              flush=True)
        for c in comms:
            lddp.lddp_comm_destroy(c)


if __name__ == "__main__":
    main()
