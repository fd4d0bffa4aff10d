"""Development tool: per (strip, warp) trace of the adiag kernel (start / end globaltimer, clock64
cycles, cycles waiting for top values and for ring back-pressure), plus the no-handoff timing.
    python tools/ad_trace.py C5 --rows 6
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("cfg")
    ap.add_argument("--rows", type=int, default=0)
    args = ap.parse_args()
    from paper_conf_ipps_kumark15_b200 import lddp
    dev = torch.device("cuda", 0)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    pb = bench.build_problem(args.cfg, dev, lddp, 1, 0, tile_rows=args.rows)
    info = json.loads(pb["plan"].info)
    print(info)
    ms, per, _, _ = bench.time_device(pb, lddp, 3, 2, dev, 1, flush)
    print("normal ms", ms)
    ns = info["strips"]
    tr = torch.zeros(ns * 4 * 6, dtype=torch.int64, device=dev)
    os.environ["LDDP_TRACE"] = f"{tr.data_ptr()}:1"
    pb = bench.build_problem(args.cfg, dev, lddp, 1, 0, tile_rows=args.rows)
    stream = torch.cuda.current_stream(dev)
    bench.do_fill(pb, lddp, stream)
    torch.cuda.synchronize()
    t = tr.cpu().numpy().reshape(ns, 4, 6).astype(np.float64)
    t0 = t[:, :, 0].min()
    st = (t[:, :, 0] - t0) / 1e3
    en = (t[:, :, 1] - t0) / 1e3
    cyc, wt, wb = t[:, :, 2], t[:, :, 3], t[:, :, 4]
    print("total us", en.max())
    for s in list(range(min(ns, 4))) + list(range(max(4, ns - 3), ns)):
        print(f"strip {s:4d} cta {int(t[s,0,5]):4d}: start " + " ".join(f"{x:8.1f}" for x in st[s]) +
              " | end " + " ".join(f"{x:8.1f}" for x in en[s]) +
              " | waittop% " + " ".join(f"{100*a/b:5.1f}" for a, b in zip(wt[s], cyc[s])) +
              " | waitbp% " + " ".join(f"{100*a/b:5.1f}" for a, b in zip(wb[s], cyc[s])))
    d = np.diff(st[:, 0])
    print("strip start lag us: mean %.2f min %.2f max %.2f" % (d.mean(), d.min(), d.max()) if len(d) else "")
    dw = st[:, 1:] - st[:, :-1]
    print("warp start lag us: mean", dw.mean(axis=0))
    dur = en - st
    print("warp duration us: mean %.1f min %.1f max %.1f" % (dur.mean(), dur.min(), dur.max()))
    print("cycles/step est (dur*1.965GHz/(n+...)):", (dur.mean() * 1965) / (info["chunks"] * 32))
    print("wait top %: mean", 100 * (wt / cyc).mean(axis=0), " bp %:", 100 * (wb / cyc).mean(axis=0))
    os.environ.pop("LDDP_TRACE")
    os.environ["LDDP_DEBUG"] = "1"
    pb = bench.build_problem(args.cfg, dev, lddp, 1, 0, tile_rows=args.rows)
    ms2, _, _, _ = bench.time_device(pb, lddp, 3, 2, dev, 1, flush)
    print("no-handoff ms", ms2, "cycles/step", ms2 * 1e-3 * 1.965e9 / (info["chunks"] * 32 + 64))


if __name__ == "__main__":
    main()
