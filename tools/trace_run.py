"""Run one wavefront fill with the in-kernel globaltimer trace (LDDP_TRACE) and summarise where
time goes per warp role: chunk compute time vs. waiting.  Development tool.

    python tools/trace_run.py --func lcs --rows 1024 --cols 1024 [--tile-rows 4]
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
    ap.add_argument("--func", default="lcs")
    ap.add_argument("--category", default="anti_diagonal")
    ap.add_argument("--rows", type=int, default=1024)
    ap.add_argument("--cols", type=int, default=1024)
    ap.add_argument("--tile-rows", type=int, default=0)
    ap.add_argument("--out", default="gpurun_out/trace.json")
    args = ap.parse_args()
    from paper_conf_ipps_kumark15_b200 import inputs, lddp
    dev = torch.device("cuda", 0)
    if args.func in ("lcs", "levenshtein"):
        a, b = inputs.gen_strings(0, args.rows, args.cols)
        ins = {"a": torch.from_numpy(a).to(dev), "b": torch.from_numpy(b).to(dev)}
    elif args.func == "dtw":
        a, b = inputs.gen_walks(0, args.rows, args.cols)
        ins = {"a": torch.from_numpy(a).to(dev), "b": torch.from_numpy(b).to(dev)}
    else:
        g = inputs.gen_image(0, args.rows, args.cols, "ramp")
        ins = {"grid": torch.from_numpy(g).to(dev)}
    outs = lddp.OUT_TABLE if args.func == "fs" else lddp.OUT_SCORE
    plan = lddp.Plan(args.func, args.category, args.rows, args.cols, outs, tile_rows=args.tile_rows)
    info = json.loads(plan.info)
    S, NQ = info["strips"], info["chunks"]
    warps = info["warps"]
    maxk = NQ + 16
    buf = torch.zeros(S * warps * maxk * 2, dtype=torch.int64, device=dev)
    t = dict(ins)
    if outs == lddp.OUT_SCORE:
        t["score"] = torch.zeros(1, dtype=torch.float32 if args.func == "dtw" else torch.int32, device=dev)
    else:
        t["table"] = torch.zeros((args.rows, args.cols), dtype=torch.uint8, device=dev)
    plan.fill(**t)   # warm
    torch.cuda.synchronize()
    os.environ["LDDP_TRACE"] = f"{buf.data_ptr()}:{maxk}"
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    plan.fill(**t)
    e.record()
    torch.cuda.synchronize()
    del os.environ["LDDP_TRACE"]
    ms = s.elapsed_time(e)
    tr = buf.cpu().numpy().reshape(S, warps, maxk, 2).astype(np.float64)
    t0 = tr[tr > 0].min()
    tr = np.where(tr > 0, tr - t0, np.nan)
    roles = [f"compute{w}" for w in range(warps - 2)] + ["loader", "storer"]
    summary = {"ms": ms, "plan": info, "roles": {}}
    for w, role in enumerate(roles):
        start, end = tr[:, w, :, 0], tr[:, w, :, 1]
        busy = np.nanmean(end - start)
        gap = np.nanmean(start[:, 1:] - end[:, :-1])
        first = np.nanmean(start[:, 0])
        last = np.nanmax(end)
        summary["roles"][role] = {"mean_chunk_ns": round(float(busy), 1), "mean_wait_ns": round(float(gap), 1),
                                  "first_start_ns_mean": round(float(first), 1), "last_end_ns": round(float(last), 1)}
    # strip start times (compute0 first chunk)
    summary["strip_start_ns"] = [round(float(x), 1) for x in tr[:, 0, 0, 0][:16]]
    summary["strip0_compute0_chunk_ns"] = [round(float(x), 1) for x in (tr[0, 0, :12, 1] - tr[0, 0, :12, 0])]
    summary["strip0_storer_chunk_ns"] = [round(float(x), 1) for x in (tr[0, warps - 1, :12, 1] - tr[0, warps - 1, :12, 0])]
    summary["strip0_storer_start_ns"] = [round(float(x), 1) for x in tr[0, warps - 1, :12, 0]]
    summary["strip1_loader_start_ns"] = [round(float(x), 1) for x in tr[min(1, S - 1), warps - 2, :12, 0]]
    summary["strip0_compute0_start_ns"] = [round(float(x), 1) for x in tr[0, 0, :12, 0]]
    summary["strip0_compute3_start_ns"] = [round(float(x), 1) for x in tr[0, warps - 3, :12, 0]]
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    with open(args.out, "w") as f:
        json.dump(summary, f, indent=1)
    np.save(args.out.replace(".json", ".npy"), tr)
    print(json.dumps(summary, indent=1))


if __name__ == "__main__":
    main()
