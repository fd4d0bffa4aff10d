"""Summarise ncu --set full captures (gpurun_out/prof_<W>.ncu-rep) into profiles/<round>_ncu.md
and profiles/traffic.json (dram read + write bytes per launch, the bench's roofline.traffic).

    python tools/profile_summary.py round1 C1 C2 C3 C4 C5
"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
        "ns": 1e-9, "us": 1e-6, "usecond": 1e-6, "ms": 1e-3, "msecond": 1e-3, "s": 1.0, "nsecond": 1e-9}
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "sm__cycles_elapsed.avg", "smsp__inst_executed.sum", "launch__grid_size", "launch__block_size",
        "launch__registers_per_thread", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__occupancy_limit_registers"]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2]


def main():
    rnd = sys.argv[1]
    names = sys.argv[2:]
    lines = [f"# ncu --set full captures, {rnd}", "",
             "One launch per workload (`-s 2 -c 1` after warm-up), `--clock-control none`, captured with",
             "`tools/gpu_bench.sh` on one B200 (numbers under ncu are cold-cache and serialised: use shares",
             "and counters, not absolute times; bench.py's CUDA-event times are the reported ones).", "",
             "| workload | kernel | grid x block | regs | duration | DRAM read | DRAM write | DRAM GB/s | ALU pipe % | FMA pipe % | top stalls |",
             "|---|---|---|---|---|---|---|---|---|---|---|"]
    traffic = {}
    for w in names:
        rep = os.path.join(ROOT, "gpurun_out", f"prof_{w}.ncu-rep")
        if not os.path.exists(rep):
            continue
        h, u, v = raw(rep)
        d = {}
        for k, unit, val in zip(h, u, v):
            try:
                d[k] = float(val.replace(",", "")) * UNIT.get(unit, 1.0)
            except ValueError:
                d[k] = val
        kname = d.get("Kernel Name", "?")
        stalls = sorted(((d[k], k.replace("smsp__pcsamp_warps_issue_stalled_", "")) for k in d
                         if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")
                         and isinstance(d[k], float)), reverse=True)
        tot = sum(s for s, _ in stalls) or 1
        st = ", ".join(f"{n} {100 * s / tot:.0f}%" for s, n in stalls[:3])
        dur = d.get("gpu__time_duration.sum", 0.0)
        rd, wr = d.get("dram__bytes_read.sum", 0.0), d.get("dram__bytes_write.sum", 0.0)
        traffic[w] = int(rd + wr)
        lines.append(f"| {w} | `{str(kname)[:60]}` | {int(d.get('launch__grid_size', 0))} x {int(d.get('launch__block_size', 0))} "
                     f"| {int(d.get('launch__registers_per_thread', 0))} | {dur * 1e3:.3f} ms | {rd / 1e6:.2f} MB | {wr / 1e6:.2f} MB "
                     f"| {(rd + wr) / dur / 1e9 if dur else 0:.0f} | {d.get('sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active', 0):.1f} "
                     f"| {d.get('sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active', 0):.1f} | {st} |")
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    with open(os.path.join(ROOT, "profiles", f"{rnd}_ncu.md"), "w") as f:
        f.write("\n".join(lines) + "\n")
    with open(os.path.join(ROOT, "profiles", "traffic.json"), "w") as f:
        json.dump(traffic, f, indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
