"""Compact summary of one ncu --set full report (run where the .ncu-rep is; writes JSON to
stdout): duration, DRAM bytes, instructions, issue / warp activity, registers, launch shape,
warp-state sample shares by stall reason, and the *stall-on-flag* share -- samples of warps
waiting on a cross-warp / cross-CTA handoff: long-scoreboard stalls within 6 instructions after a
strong (relaxed / acquire / volatile) global load, mbarrier try-waits, plus every backoff sleep.
Measurement tool (SURVEY §8(d) evidence counters).

    python tools/ncu_summary.py report.ncu-rep > summary.json
"""
import csv
import io
import json
import subprocess
import sys

RAW = {
    "gpu__time_duration.sum": "duration",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "smsp__inst_executed.sum": "inst_executed",
    "smsp__issue_active.avg.pct_of_peak_sustained_active": "issue_active_pct",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "warps_active_pct",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed": "sm_throughput_pct",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed": "dram_throughput_pct",
    "launch__registers_per_thread": "registers",
    "launch__grid_size": "grid",
    "launch__block_size": "block",
    "sm__cycles_active.avg": "sm_cycles_active",
    "gpc__cycles_elapsed.max": "cycles_elapsed",
}


def ncu(rep, *args):
    return subprocess.run(["ncu", "-i", rep, *args], capture_output=True, text=True).stdout


def main():
    rep = sys.argv[1]
    rows = list(csv.reader(io.StringIO(ncu(rep, "--page", "raw", "--csv"))))
    out = {"report": rep.split("/")[-1]}
    if len(rows) >= 3:
        h, units, v = rows[0], rows[1], rows[2]
        for i, name in enumerate(h):
            if name == "Kernel Name":
                out["kernel"] = v[i][:160]
            if name in RAW:
                out[RAW[name]] = f"{v[i]} {units[i]}".strip()
    src = list(csv.reader(io.StringIO(ncu(rep, "--page", "source", "--csv", "--print-source", "sass"))))
    if len(src) > 2:
        h = src[1]
        data = src[2:]
        isrc = h.index("Source")
        iss = h.index("Warp Stall Sampling (All Samples)")
        reasons = [c for c in h if c.startswith("stall_") and "Not Issued" not in c]
        ir = {c: h.index(c) for c in reasons}
        tot = sum(int(r[iss] or 0) for r in data)
        agg = {c: sum(int(r[ir[c]] or 0) for r in data) for c in reasons}
        out["samples"] = tot
        out["stall_shares"] = {c[6:]: round(n / max(tot, 1), 4) for c, n in sorted(agg.items(), key=lambda x: -x[1]) if n}
        flag = 0
        since = 99
        for r in data:
            s = r[isrc]
            if ("LDG" in s or "LD.E" in s or " LD." in s) and "STRONG" in s:
                since = 0
            else:
                since += 1
            if since <= 6 and "stall_long_sb" in ir:
                flag += int(r[ir["stall_long_sb"]] or 0)
            if "TRYWAIT" in s or "SYNCS.PHASECHK" in s:
                flag += int(r[iss] or 0)
        flag += agg.get("stall_sleep", 0)
        out["stall_on_flag_share"] = round(flag / max(tot, 1), 4)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
