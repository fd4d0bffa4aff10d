"""Write profiles/round2_ncu.md and profiles/traffic.json from the ncu summaries of
tools/gpu_round2_prof.sh (gpurun_out/r2/prof_*.json, tools/ncu_summary.py).  Measurement tool.

    python tools/make_ncu_md.py gpurun_out/r2
"""
import glob
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
WORKLOAD = {"c1": "C1", "c2": "C2", "c3": "C3", "c4": "C4", "c5": "C5", "c6": "C6", "c7": "C7", "c8": "C8"}


def num(s):
    try:
        v, u = s.split(" ", 1)
    except (ValueError, AttributeError):
        return None, ""
    return float(v), u


def to_ms(s):
    v, u = num(s)
    if v is None:
        return None
    return v * {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0,
                "s": 1e3, "second": 1e3}.get(u.strip(), 1.0)


def to_bytes(s):
    v, u = num(s)
    if v is None:
        return None
    return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u.strip(), 1)


def main():
    src = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "gpurun_out", "r2")
    rows = []
    traffic = {}
    tpath = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tpath):
        traffic = json.load(open(tpath))
    for f in sorted(glob.glob(os.path.join(src, "prof_*.json"))):
        try:
            d = json.load(open(f))
        except Exception:
            continue
        if "kernel" not in d:
            continue
        name = os.path.basename(f)[5:-5]
        rd, wr = to_bytes(d.get("dram_read")), to_bytes(d.get("dram_write"))
        wl = WORKLOAD.get(name.split("_")[0])
        if wl and rd is not None and wr is not None:
            traffic[wl] = int(rd + wr)
        rows.append((name, d, rd, wr))
    with open(tpath, "w") as fh:
        json.dump(traffic, fh, indent=1)
    out = ["# Round 2 ncu captures (one B200, `ncu --set full --clock-control none`, one launch each)", "",
           "Written by `tools/make_ncu_md.py` from `tools/gpu_round2_prof.sh` (summaries by",
           "`tools/ncu_summary.py`).  *stall on flag* = warp-state samples waiting on a handoff: long-",
           "scoreboard stalls right after a strong (relaxed / acquire) global load, mbarrier try-waits and",
           "backoff sleeps.  ncu times are cold-cache and serialised: compare shares, not absolutes, with",
           "the bench line.", "",
           "| capture | kernel | ms | DRAM read + write | inst | issue active | warps active | regs | grid × block | stall on flag | top stall reasons |",
           "|---|---|---|---|---|---|---|---|---|---|---|"]
    for name, d, rd, wr in rows:
        dur = to_ms(d.get("duration", "")) or 0.0
        inst, _ = num(d.get("inst_executed", ""))
        top = ", ".join(f"{k} {v:.0%}" for k, v in list(d.get("stall_shares", {}).items())[:3])
        byt = f"{(rd or 0) / 1e9:.3f} + {(wr or 0) / 1e9:.3f} GB" if rd is not None else "—"
        out.append(f"| {name} | `{d['kernel'][:70]}` | {dur:.4f} | {byt} | {inst / 1e6:.1f} M | "
                   f"{d.get('issue_active_pct', '—')} | {d.get('warps_active_pct', '—')} | "
                   f"{num(d.get('registers', ''))[0] or '—'} | {d.get('grid', '')} × {d.get('block', '')} | "
                   f"{d.get('stall_on_flag_share', 0):.1%} | {top} |")
    with open(os.path.join(ROOT, "profiles", "round2_ncu.md"), "w") as fh:
        fh.write("\n".join(out) + "\n")
    print("\n".join(out))


if __name__ == "__main__":
    main()
