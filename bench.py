#!/usr/bin/env python
"""bench.py -- GCUPS of the B200-native LDDP-Plus fill (BASELINE.json metric) on N GPUs.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload C5] [--impl ours|reference]
    (N > 1: python -m torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1 ... bench.py --gpus N)

A step = one whole dependency-ordered fill (all §8(a) rows: plan already made, inputs resident,
one persistent kernel) of the named workload.  Default workload C5 = LCS 100000 x 100000, the
BASELINE config quoted "at 1/2/4/8 B200"; on N GPUs it runs as N column strips (strong
scaling, lddp_fill_multi: peer stores over NVLink).  At N = 1 the other configs C1-C4 are also
measured and reported under "configs" of the same JSON line.

Timing: W untimed warm-up steps, then exactly K steps bracketed by barrier + synchronize; each
step's fill is bracketed by CUDA events on the launching stream, and a 256 MiB buffer (> the
126 MB L2) is overwritten between steps (outside the events); reported time = max over ranks of
the summed event times.  `e2e` is the same metric through the host-buffer C-ABI call
(lddp_fill_host: pinned H2D of the inputs, fill, D2H of the score, synchronize).
"""
import argparse
import hashlib
import json
import os
import sys
import threading
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
from configs import CONFIGS  # noqa: E402

PEAKS_FILE = os.path.join(ROOT, "MEASURED_PEAKS.json")
FALLBACK_PEAKS = {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0, "_source": "fallback (B200_PROFILING.md)"}
# Algorithmic work per cell on the binding pipe: LCS = compare + 3-way max on
# the INT ALU pipe; DTW = subtract + add on the FP32 (FMA) pipe; FS = 4 mul + 5 add on the FMA
# pipe; min-path = the 4-byte cost read from HBM.
ALU_OPS_PER_CELL = {"lcs": 2, "levenshtein": 3, "dtw": 2, "fs": 9}
PIPE_LANES_PER_SM_CLK = 64            # ALU pipe and FMA pipe: 16 lanes/clk per SMSP x 4
NUM_SMS = 148


def load_peaks():
    try:
        with open(PEAKS_FILE) as f:
            p = json.load(f)
        p["_source"] = "measured (MEASURED_PEAKS.json)"
        return p
    except Exception:
        return dict(FALLBACK_PEAKS)


def traffic_for(workload):
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            return json.load(f).get(workload)
    except Exception:
        return None


class ClockSampler:
    """Samples SM clock + throttle reasons with NVML every 10 ms."""

    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
               0x8: "hw_slowdown", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
               0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}

    def __init__(self, index):
        self.samples = []
        self.ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception:
            self.max_mhz = None
        self._stop = threading.Event()
        self._t = None

    def _run(self):
        while not self._stop.is_set():
            try:
                mhz = self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM)
                rs = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                self.samples.append((time.time(), mhz, rs))
            except Exception:
                pass
            time.sleep(0.01)

    def start(self):
        if self.ok:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()

    def stop(self):
        if self._t:
            self._stop.set()
            self._t.join()

    def summary(self, t0, t1):
        win = [s for s in self.samples if t0 <= s[0] <= t1] or self.samples
        if not win:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": [], "samples": 0}
        mhz = sorted(s[1] for s in win)
        bits = 0
        for s in win:
            bits |= s[2]
        reasons = [name for bit, name in self.REASONS.items() if bits & bit]
        return {"sm_mhz": mhz[len(mhz) // 2], "sm_max_mhz": self.max_mhz, "reasons": reasons,
                "samples": len(win)}


def _coll_dev(dev):
    """Device for collective tensors: the GPU with NCCL, the CPU with a gloo test group."""
    return torch.device("cpu") if os.environ.get("LDDP_BENCH_BACKEND", "nccl") != "nccl" else dev


def dist_info():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def refs():
    with open(os.path.join(ROOT, "tests", "golden", "bench_refs.json")) as f:
        return json.load(f)["configs"]


def sha(t):
    return hashlib.sha256(np.ascontiguousarray(t).tobytes()).hexdigest()


# ------------------------------------------------------------------------------------------
def build_problem(name, dev, lddp, world, rank, tile_rows=0):
    cfg = CONFIGS[name]
    x = cfg["make"](0)
    func, cat = cfg["func"], cfg["category"]
    rows, cols = cfg["rows"], cfg["cols"]
    outs = {"lcs": lddp.OUT_SCORE, "dtw": lddp.OUT_SCORE, "fs": lddp.OUT_TABLE,
            "minpath3": lddp.OUT_SCORE | lddp.OUT_LAST_ROW}[func]
    plan = lddp.Plan(func, cat, rows, cols, outs, device=dev.index, tile_rows=tile_rows)
    t = {}
    h2d = 0
    if "a" in x:
        t["a"] = torch.from_numpy(x["a"]).to(dev)
        t["b"] = torch.from_numpy(x["b"]).to(dev)
        h2d = x["a"].nbytes + x["b"].nbytes
    else:
        t["grid"] = torch.from_numpy(x["grid"]).to(dev)
        h2d = x["grid"].nbytes
    cell_dt = torch.float32 if func == "dtw" else torch.int32
    if outs & lddp.OUT_SCORE:
        t["score"] = torch.zeros(1, dtype=cell_dt, device=dev)
    if outs & lddp.OUT_LAST_ROW:
        t["last_row"] = torch.zeros(cols, dtype=cell_dt, device=dev)
    if outs & lddp.OUT_TABLE:
        t["table"] = torch.zeros((rows, cols), dtype=torch.uint8, device=dev)
    comm = None
    if world > 1:
        import torch.distributed as dist
        comm = lddp.lddp_comm_create(plan.handle, world, rank)
        handles = [None] * world
        dist.all_gather_object(handles, lddp.lddp_comm_handle(comm))
        lddp.lddp_comm_connect(comm, handles[rank + 1] if rank + 1 < world else None,
                               handles[rank - 1] if rank > 0 else None)
        dist.barrier()
    return {"cfg": cfg, "x": x, "plan": plan, "t": t, "comm": comm, "h2d": h2d, "outs": outs}


def do_fill(pb, lddp, stream):
    inp, out = pb["plan"].io(**pb["t"])
    if pb["comm"] is None:
        lddp.lddp_fill(pb["plan"].handle, inp, out, pb["plan"].ws.data_ptr(), stream.cuda_stream)
    else:
        lddp.lddp_fill_multi(pb["plan"].handle, inp, out, pb["plan"].ws.data_ptr(), pb["comm"],
                             stream.cuda_stream)


def time_device(pb, lddp, steps, warmup, dev, world, flush):
    stream = torch.cuda.current_stream(dev)
    for _ in range(warmup):
        do_fill(pb, lddp, stream)
    pb["plan"].check()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
    torch.cuda.synchronize(dev)
    t0 = time.time()
    for k in range(steps):
        flush.zero_()
        ev[k][0].record(stream)
        do_fill(pb, lddp, stream)
        ev[k][1].record(stream)
    torch.cuda.synchronize(dev)
    t1 = time.time()
    if world > 1:
        dist.barrier()
    pb["plan"].check()
    ms = [s.elapsed_time(e) for s, e in ev]
    total = sum(ms)
    if world > 1:
        tt = torch.tensor([total], dtype=torch.float64, device=_coll_dev(dev))
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        total = float(tt.item())
    return total / steps, ms, t0, t1


def time_e2e(pb, lddp, steps, dev, world):
    """Same metric through the public host-buffer path: pinned H2D of this step's inputs, the
    fill, D2H of the step's result (score), synchronize."""
    cfg, x = pb["cfg"], pb["x"]
    host_in = {k: torch.from_numpy(v).pin_memory() for k, v in x.items()}
    cell_dt = torch.float32 if cfg["func"] == "dtw" else torch.int32
    res = torch.zeros(1, dtype=cell_dt).pin_memory()
    d2h = 4
    if world == 1:
        plan = pb["plan"]
        tbl = None
        if pb["outs"] & lddp.OUT_TABLE:
            tbl = torch.zeros((cfg["rows"], cfg["cols"]), dtype=torch.uint8).pin_memory()
            d2h = tbl.numel()
        lr = None
        if pb["outs"] & lddp.OUT_LAST_ROW:
            lr = torch.zeros(cfg["cols"], dtype=cell_dt).pin_memory()
            d2h += lr.numel() * 4
        inp, out = plan.io(a=host_in.get("a"), b=host_in.get("b"), grid=host_in.get("grid"),
                           score=res if pb["outs"] & lddp.OUT_SCORE else None, last_row=lr, table=tbl)
        if tbl is not None:
            d2h -= 4
        stream = torch.cuda.current_stream(dev)
        lddp.lddp_fill_host(plan.handle, inp, out, stream.cuda_stream)   # warm staging buffers
        t0 = time.perf_counter()
        for _ in range(steps):
            lddp.lddp_fill_host(plan.handle, inp, out, stream.cuda_stream)
        dt = (time.perf_counter() - t0) / steps
        return dt, pb["h2d"], d2h
    # multi-GPU: each rank copies the inputs it reads, fills its strip, reads the score back
    import torch.distributed as dist
    stream = torch.cuda.current_stream(dev)
    da, db = pb["t"]["a"], pb["t"]["b"]
    dist.barrier()
    t0 = time.perf_counter()
    for _ in range(steps):
        da.copy_(host_in["a"], non_blocking=True)
        db.copy_(host_in["b"], non_blocking=True)
        do_fill(pb, lddp, stream)
        res.copy_(pb["t"]["score"], non_blocking=True)
        torch.cuda.synchronize(dev)
    dt = (time.perf_counter() - t0) / steps
    tt = torch.tensor([dt], dtype=torch.float64, device=_coll_dev(dev))
    dist.all_reduce(tt, op=dist.ReduceOp.MAX)
    return float(tt.item()), pb["h2d"], 4


def check_result(name, pb):
    ref = refs().get(name)
    if ref is None:
        return {"checked": False}
    t = pb["t"]
    ok = True
    got = {}
    if "score" in ref and "score" in t:
        s = t["score"].cpu().numpy()[0]
        got["score"] = float(s) if CONFIGS[name]["func"] == "dtw" else int(s)
        if CONFIGS[name]["func"] == "dtw":
            ok &= abs(got["score"] - ref["score"]) <= 1e-5 * abs(ref["score"])
        else:
            ok &= got["score"] == ref["score"]
    if "last_row_sha256" in ref and "last_row" in t:
        ok &= sha(t["last_row"].cpu().numpy()) == ref["last_row_sha256"]
    if "image_sha256" in ref and "table" in t:
        ok &= sha(t["table"].cpu().numpy()) == ref["image_sha256"]
    return {"checked": True, "match": bool(ok), "vs": "tests/golden/bench_refs.json (oracle, seed 0)", **got}


def gather_parity(name, pb, world, rank):
    """The score lives on the last rank (column strips): check there, share with rank 0."""
    res = check_result(name, pb) if rank == world - 1 else {"checked": False}
    if world > 1:
        import torch.distributed as dist
        box = [res]
        dist.broadcast_object_list(box, src=world - 1)
        res = box[0]
    return res


def roofline(name, ms_per_step, peaks, world, clock_mhz):
    cfg = CONFIGS[name]
    cells = cfg["rows"] * cfg["cols"]
    t = ms_per_step / 1e3
    if cfg["func"] == "minpath3":
        alg_bytes = cells * 4 + cfg["cols"] * 4 + 4
        achieved = alg_bytes / t / 1e9
        peak = peaks.get("hbm_gbs", 6650.0) * world
        return {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                "frac": round(achieved / peak, 4), "traffic": traffic_for(name),
                "algorithmic_bytes_per_cell": 4, "peak_source": peaks.get("_source")}
    ops = ALU_OPS_PER_CELL[cfg["func"]]
    mhz = peaks.get("sm_max_mhz", 1965.0)
    peak = NUM_SMS * PIPE_LANES_PER_SM_CLK * mhz * 1e6 * world / 1e12
    achieved = cells * ops / t / 1e12
    pipe = "FMA (FP32)" if cfg["func"] in ("dtw", "fs") else "ALU (INT)"
    return {"bound": "alu", "achieved": round(achieved, 3), "peak": round(peak, 2), "unit": "Tops/s",
            "frac": round(achieved / peak, 4), "traffic": traffic_for(name),
            "pipe": pipe, "algorithmic_ops_per_cell": ops,
            "peak_derivation": f"{NUM_SMS} SMs x {PIPE_LANES_PER_SM_CLK} lanes/clk x {mhz:.0f} MHz x {world} GPU",
            "sm_mhz_during_run": clock_mhz}


def cpu_baseline(name):
    """The oracle as it stands, single-threaded, on a bounded sample of the workload."""
    import oracle
    cfg = CONFIGS[name]
    x = cfg["make"](0)
    func = cfg["func"]
    t0 = time.perf_counter()
    if func == "lcs":
        rows = min(cfg["rows"], max(1, int(2.5e9 // cfg["cols"])))
        oracle.lcs(x["a"][:rows], x["b"])
        cells, sample = rows * cfg["cols"], f"first {rows} rows x all {cfg['cols']} columns"
    elif func == "dtw":
        rows = min(cfg["rows"], max(1, int(1.0e9 // cfg["cols"])))
        oracle.dtw(x["a"][:rows], x["b"])
        cells, sample = rows * cfg["cols"], f"first {rows} rows x all {cfg['cols']} columns"
    elif func == "fs":
        oracle.fs(x["grid"])
        cells, sample = cfg["rows"] * cfg["cols"], "whole image"
    else:
        oracle.minpath3(x["grid"])
        cells, sample = cfg["rows"] * cfg["cols"], "whole grid"
    dt = time.perf_counter() - t0
    return {"value": round(cells / dt / 1e9, 4), "unit": "GCUPS", "cores": 1, "kind": "oracle",
            "sample": sample, "seconds": round(dt, 2)}


def measure(name, lddp, dev, world, rank, steps, warmup, flush, peaks, sampler, with_e2e=True,
            tile_rows=0):
    pb = build_problem(name, dev, lddp, world, rank, tile_rows=tile_rows)
    ms, per, t0, t1 = time_device(pb, lddp, steps, warmup, dev, world, flush)
    cfg = CONFIGS[name]
    cells = cfg["rows"] * cfg["cols"]
    clocks = sampler.summary(t0, t1) if sampler else None
    out = {"value": round(cells / (ms / 1e3) / 1e9, 3), "ms_per_step": round(ms, 4),
           "ms_min": round(min(per), 4), "ms_max": round(max(per), 4),
           "roofline": roofline(name, ms, peaks, world, clocks["sm_mhz"] if clocks else None),
           "parity": gather_parity(name, pb, world, rank),
           "plan": json.loads(pb["plan"].info), "clocks": clocks}
    if with_e2e:
        dt, bi, bo = time_e2e(pb, lddp, max(3, min(steps, 10)), dev, world)
        out["e2e"] = {"value": round(cells / dt / 1e9, 3), "unit": "GCUPS", "h2d_bytes_per_step": bi,
                      "d2h_bytes_per_step": bo}
    if pb["comm"] is not None:
        lddp.lddp_comm_destroy(pb["comm"])
    return out


def run_reference(args, world, rank):
    """--impl reference: the oracle (plain CPU fill) as it stands, on the host cores."""
    if rank != 0:
        return
    name = args.workload
    vals = []
    for _ in range(args.warmup):
        pass  # the oracle has no warm-up state; warm-up steps are skipped
    samples = []
    for _ in range(args.steps):
        cb = cpu_baseline(name)
        vals.append(cb["value"])
        samples.append(cb)
    v = float(np.median(vals))
    cfg = CONFIGS[name]
    line = {"impl": "reference", "metric": "GCUPS (cell updates/s)", "value": v, "unit": "GCUPS",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": None, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "int32" if cfg["func"] != "dtw" else "f32",
            "data": "synthetic (seed 0)",
            "config": {"workload": name, "desc": cfg["desc"], "rows": cfg["rows"], "cols": cfg["cols"]},
            "cpu_baseline": {"value": v, "unit": "GCUPS", "cores": 1, "kind": "oracle",
                             "sample": samples[0]["sample"] + " (each step)"},
            "e2e": {"value": v, "unit": "GCUPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--workload", default="C5", choices=sorted(CONFIGS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-others", action="store_true", help="skip C1-C4 at N=1")
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--tile-rows", type=int, default=0)
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    world, rank, local = dist_info()
    if args.impl == "reference":
        run_reference(args, world, rank)
        return

    from paper_conf_ipps_kumark15_b200 import lddp

    # Test hooks (not used by the driver): LDDP_BENCH_SAME_DEVICE=1 puts every rank on cuda:0 and
    # LDDP_BENCH_BACKEND=gloo uses a CPU process group -- exercises the cross-process CUDA-IPC
    # window path on a single GPU (set LDDP_GRID_CTAS so all ranks' kernels are co-resident).
    if os.environ.get("LDDP_BENCH_SAME_DEVICE") == "1":
        local = 0
    dev = torch.device("cuda", local)
    torch.cuda.set_device(dev)
    if world > 1:
        import torch.distributed as dist
        backend = os.environ.get("LDDP_BENCH_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    peaks = load_peaks()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    sampler = ClockSampler(local)
    sampler.start()
    head = measure(args.workload, lddp, dev, world, rank, args.steps, args.warmup, flush, peaks,
                   sampler, tile_rows=args.tile_rows)
    others = {}
    if world == 1 and not args.no_others:
        for name in ("C1", "C2", "C3", "C4"):
            if name == args.workload:
                continue
            r = measure(name, lddp, dev, 1, 0, max(5, args.steps // 2), args.warmup, flush, peaks, sampler,
                        with_e2e=False)
            others[name] = {"desc": CONFIGS[name]["desc"], "value": r["value"], "unit": "GCUPS",
                            "ms_per_step": r["ms_per_step"], "roofline": r["roofline"],
                            "parity": r["parity"], "plan": r["plan"]}
            torch.cuda.empty_cache()
    sampler.stop()
    cpu = None
    if world == 1 and rank == 0 and not args.no_cpu:
        cpu = cpu_baseline(args.workload)
    if rank == 0:
        cfg = CONFIGS[args.workload]
        line = {"metric": "GCUPS (cell updates/s)", "value": head["value"], "unit": "GCUPS",
                "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
                "ms_per_step": head["ms_per_step"], "higher_is_better": True,
                "scaling": "strong",
                "vs_baseline": None, "dtype": "f32" if cfg["func"] == "dtw" else "int32",
                "data": "synthetic (seed 0, DESIGN.md §4 recipe)",
                "config": {"workload": args.workload, "desc": cfg["desc"], "rows": cfg["rows"],
                           "cols": cfg["cols"], "func": cfg["func"], "category": cfg["category"],
                           "parallelism": f"column strips x{world}" if world > 1 else "single GPU",
                           "l2": "256 MiB buffer overwritten between timed steps (outside the events)",
                           "timing": "CUDA events around each fill on its stream, summed over K steps, max over ranks"},
                "clocks": head["clocks"], "e2e": head.get("e2e"),
                "gpu_launches": args.steps * world,
                "roofline": head["roofline"], "cpu_baseline": cpu, "parity": head["parity"],
                "plan": head["plan"], "ms_min": head["ms_min"], "ms_max": head["ms_max"],
                "configs": others}
        print(json.dumps(line), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
