"""Summarise an ncu --page source --csv --print-source sass export: instructions with their
executions per unit and stall-reason samples (development tool).

    python tools/ncu_src.py export.csv --units 16777216 [--min-frac 0.004] [--lo 1400 --hi 1890]
"""
import argparse
import csv

REASONS = ["stall_long_sb", "stall_short_sb", "stall_wait", "stall_selected", "stall_math", "stall_mio",
           "stall_lg", "stall_branch_resolving", "stall_no_inst", "stall_dispatch", "stall_not_selected",
           "stall_barrier", "stall_membar", "stall_drain", "stall_misc", "stall_sleep"]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("csv")
    ap.add_argument("--units", type=float, default=1.0, help="divide execution counts by this")
    ap.add_argument("--min-frac", type=float, default=0.004)
    ap.add_argument("--lo", default=None)
    ap.add_argument("--hi", default=None)
    args = ap.parse_args()
    rows = list(csv.reader(open(args.csv)))
    h = rows[1]
    data = rows[2:]
    ia, isrc = h.index("Address"), h.index("Source")
    iss, iex = h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
    ir = {r: h.index(r) for r in REASONS if r in h}
    tot = sum(int(r[iss]) for r in data)
    agg = {r: 0 for r in ir}
    for r in data:
        for k, i in ir.items():
            agg[k] += int(r[i] or 0)
    print("total samples", tot, {k: round(v / max(tot, 1), 3) for k, v in sorted(agg.items(), key=lambda x: -x[1]) if v})
    lo = int(args.lo, 16) if args.lo else None
    hi = int(args.hi, 16) if args.hi else None
    for r in data:
        a = int(r[ia], 16) & 0xFFFFF
        if lo is not None and not (lo <= a <= hi):
            continue
        s = int(r[iss])
        if lo is None and s < tot * args.min_frac:
            continue
        top = sorted(((int(r[i] or 0), k[6:]) for k, i in ir.items()), reverse=True)[:2]
        print(f"{a:05x} {int(r[iex]) / args.units:7.3f} {s:6d} {' '.join(f'{k}:{v}' for v, k in top if v):28s} {r[isrc][:80]}")


if __name__ == "__main__":
    main()
