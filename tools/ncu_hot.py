"""Summarise an ncu report: duration, top stall reasons, and the hottest SASS instructions with
their per-instruction stall samples (needs -lineinfo builds).  Development tool.

    python tools/ncu_hot.py gpurun_out/prof.ncu-rep [--top 40] [--range lo hi]
"""
import argparse
import csv
import io
import subprocess


def ncu_csv(rep, *args):
    out = subprocess.run(["ncu", "-i", rep, *args, "--csv"], capture_output=True, text=True).stdout
    return list(csv.reader(io.StringIO(out)))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("--top", type=int, default=40)
    ap.add_argument("--context", type=int, default=0)
    args = ap.parse_args()
    raw = ncu_csv(args.rep, "--page", "raw")
    h, v = raw[0], raw[2]
    want = ["gpu__time_duration.sum", "sm__cycles_elapsed.avg", "smsp__inst_executed.sum",
            "dram__bytes_read.sum", "dram__bytes_write.sum", "launch__grid_size",
            "sm__warps_active.avg.pct_of_peak_sustained_active"]
    for k, val in zip(h, v):
        if k in want:
            print(f"{k:60s} {val}")
    stalls = []
    for k, val in zip(h, v):
        if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued"):
            try:
                stalls.append((float(val.replace(",", "")), k.replace("smsp__pcsamp_warps_issue_stalled_", "")))
            except ValueError:
                pass
    tot = sum(s for s, _ in stalls) or 1
    print("stall samples:", ", ".join(f"{n} {100 * s / tot:.1f}%" for s, n in sorted(stalls, reverse=True)[:8]))
    src = ncu_csv(args.rep, "--page", "source", "--print-source", "sass")
    hdr = src[1]
    rows = src[2:]
    isrc, iss, iex = hdr.index("Source"), hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Instructions Executed")
    order = sorted(range(len(rows)), key=lambda i: -int(rows[i][iss] or 0))[: args.top]
    tot_s = sum(int(r[iss] or 0) for r in rows) or 1
    for i in sorted(order):
        r = rows[i]
        print(f"{i:6d} {int(r[iss] or 0):8d} {100 * int(r[iss] or 0) / tot_s:5.1f}% ex={r[iex]:>10s}  {r[isrc].strip()[:90]}")


if __name__ == "__main__":
    main()
