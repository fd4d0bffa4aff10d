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
import subprocess
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
LATENCY_FILE = os.path.join(ROOT, "profiles", "round2_latency.json")   # tools/micro/lat2.cu on B200
# Algorithmic work per cell, SURVEY.md §8(d) "Algorithmic work per cell": (ops, pipe).  The INT
# ALU pipe has 64 lanes/clk/SM (16 per SM sub-partition), the FP32 FMA pipe 128.
WORK = {"lcs": (3, "alu"), "levenshtein": (3, "alu"), "dtw": (3, "fma"), "fs": (11, "fma"),
        "minpath3": (2, "alu"), "min2plus": (2, "alu"), "diagmaxplus": (2, "alu")}
LANES = {"alu": 64, "fma": 128}
# Algorithmic HBM bytes per cell (inputs read once, outputs written once; the table is virtual)
HBM_PER_CELL = {"fs": 2.0, "minpath3": 4.0, "min2plus": 4.0, "diagmaxplus": 4.0}
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
            "minpath3": lddp.OUT_SCORE | lddp.OUT_LAST_ROW, "min2plus": lddp.OUT_SCORE | lddp.OUT_LAST_ROW,
            "diagmaxplus": lddp.OUT_LAST_ROW | lddp.OUT_LAST_COL}[func]
    plan = lddp.Plan(func, cat, cfg.get("img_rows", rows), cols, outs, device=dev.index, tile_rows=tile_rows,
                     param_c=cfg.get("param_c", 1), batch=cfg.get("batch", 0))
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
    if outs & lddp.OUT_LAST_COL:
        t["last_col"] = torch.zeros(rows, dtype=cell_dt, device=dev)
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
        lr = lc = None
        if pb["outs"] & lddp.OUT_LAST_ROW:
            lr = torch.zeros(cfg["cols"], dtype=cell_dt).pin_memory()
            d2h += lr.numel() * 4
        if pb["outs"] & lddp.OUT_LAST_COL:
            lc = torch.zeros(cfg["rows"], dtype=cell_dt).pin_memory()
            d2h += lc.numel() * 4
        if not pb["outs"] & lddp.OUT_SCORE:
            d2h -= 4
        inp, out = plan.io(a=host_in.get("a"), b=host_in.get("b"), grid=host_in.get("grid"),
                           score=res if pb["outs"] & lddp.OUT_SCORE else None, last_row=lr, last_col=lc,
                           table=tbl)
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
    if "last_col_sha256" in ref and "last_col" in t:
        ok &= sha(t["last_col"].cpu().numpy()) == ref["last_col_sha256"]
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


def load_latency():
    try:
        with open(LATENCY_FILE) as f:
            return json.load(f)
    except Exception:   # a-priori constants of SURVEY.md §8(d)
        return {"lcs_cell": 4.5, "levenshtein_cell": 9.0, "dtw_cell": 10.0, "fs_cell": 28.0, "minpath_row": 11.0,
                "_source": "a-priori (SURVEY.md 8(d))"}


def roofline(name, ms_per_step, peaks, world, clock_mhz):
    """the roofline time is max(T_work, T_span, T_mem); the binding term is
    reported with its achieved / peak / frac, the others beside it."""
    cfg = CONFIGS[name]
    func, cat = cfg["func"], cfg["category"]
    H, W = cfg.get("img_rows", cfg["rows"]), cfg["cols"]   # one image's shape (span); cells = the whole batch
    cells = cfg["rows"] * W
    t = ms_per_step / 1e3
    mhz = peaks.get("sm_max_mhz", 1965.0)
    ops, pipe = WORK[func]
    peak_ops = NUM_SMS * LANES[pipe] * mhz * 1e6 * world          # lane-ops / s
    t_work = cells * ops / peak_ops
    lat = load_latency()
    key = {"lcs": "lcs_cell", "levenshtein": "levenshtein_cell", "dtw": "dtw_cell", "fs": "fs_cell"}.get(func, "minpath_row")
    cyc = float(lat[key])
    path = {"anti_diagonal": H + W - 1, "knight_move": 2 * (H - 1) + W, "prev_row": H,
            "inverted_l": min(H, W)}[cat]                     # cells on the longest dependency path
    t_span = path * cyc / (mhz * 1e6)
    hbm_bytes = cells * HBM_PER_CELL.get(func, 0.0) + 4 * (cfg["rows"] + W)
    peak_bw = peaks.get("hbm_gbs", 6650.0) * 1e9 * world
    t_mem = hbm_bytes / peak_bw
    terms = {"work": t_work, "span": t_span, "mem": t_mem}
    bound = max(terms, key=terms.get)
    out = {"traffic": traffic_for(name), "sm_mhz_during_run": clock_mhz,
           "terms_ms": {k: round(v * 1e3, 4) for k, v in terms.items()},
           "frac_by_term": {k: round(v / t, 4) for k, v in terms.items()},
           "work_per_cell": f"{ops} {'INT ALU' if pipe == 'alu' else 'FP32 FMA'} ops (SURVEY 8(d))",
           "work_peak": f"{NUM_SMS} SMs x {LANES[pipe]} lanes/clk x {mhz:.0f} MHz x {world} GPU = {peak_ops / 1e12:.2f} T lane-ops/s",
           "span_model": f"{path} dependent cells x {cyc:.2f} cycles ({lat.get('how', lat.get('_source', ''))})",
           "hbm_bytes_per_step": hbm_bytes, "hbm_peak_source": peaks.get("_source")}
    if bound == "mem":
        ach = hbm_bytes / t / 1e9
        out.update({"bound": "hbm", "achieved": round(ach, 1), "peak": round(peak_bw / 1e9, 1), "unit": "GB/s",
                    "frac": round(ach / (peak_bw / 1e9), 4)})
    elif bound == "work":
        ach = cells * ops / t / 1e12
        out.update({"bound": "alu" if pipe == "alu" else "fma", "achieved": round(ach, 3),
                    "peak": round(peak_ops / 1e12, 2), "unit": "Tops/s", "frac": round(ach / (peak_ops / 1e12), 4)})
    else:
        ach = cells / t / 1e9
        pk = cells / t_span / 1e9
        out.update({"bound": "span", "achieved": round(ach, 3), "peak": round(pk, 1), "unit": "GCUPS",
                    "frac": round(ach / pk, 4)})
    return out


def host_info():
    model = ""
    try:
        for line in subprocess.run(["lscpu"], capture_output=True, text=True).stdout.splitlines():
            if line.startswith("Model name:"):
                model = line.split(":", 1)[1].strip()
    except Exception:
        pass
    return {"nproc": os.cpu_count(), "cpu_model": model}


def cpu_baseline(name):
    """The oracle as it stands, single-threaded and pinned to one core (os.sched_setaffinity, the
    in-process equivalent of taskset -c), on a bounded sample of the workload."""
    import oracle
    cfg = CONFIGS[name]
    x = cfg["make"](0)
    func = cfg["func"]
    try:
        old_aff = os.sched_getaffinity(0)
        core = min(old_aff)
        os.sched_setaffinity(0, {core})
    except Exception:
        old_aff, core = None, None
    try:
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
            ir = cfg.get("img_rows", cfg["rows"])
            oracle.fs(x["grid"][:ir])
            cells, sample = ir * cfg["cols"], "one whole image"
        elif func in ("min2plus", "diagmaxplus"):
            rows = min(cfg["rows"], 8192)
            getattr(oracle, func)(x["grid"][:rows], cfg.get("param_c", 1))
            cells, sample = rows * cfg["cols"], f"first {rows} rows x all {cfg['cols']} columns"
        else:
            oracle.minpath3(x["grid"])
            cells, sample = cfg["rows"] * cfg["cols"], "whole grid"
        dt = time.perf_counter() - t0
    finally:
        if old_aff is not None:
            os.sched_setaffinity(0, old_aff)
    return {"value": round(cells / dt / 1e9, 4), "unit": "GCUPS", "cores": 1, "kind": "oracle",
            "sample": sample, "seconds": round(dt, 2), "pinned_core": core, **host_info()}


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


def scaling_model(ms1, plan, cols):
    """column strips of n/P columns per rank.  Rank g's strip s needs rank g-1's
    whole right column of strip s (its last chunk), so start(g, s) = s*L + g*(NQ/P + 2E) chunks
    and the fill ends at (S-1)*L + P*(NQ/P + 2E) = T(1) + 2E(P-1) chunks: strong scaling is
    capped at ~1x by the lane-systolic sweep (every row strip crosses all n columns one chunk at a
    time, at the same per-chunk cost on any GPU count).  The per-chunk time t and the strip lag L
    (2E + 1 chunks of structure + ~0.9 chunk of handoff latency, tools/l16_trace.py) are
    calibrated on the measured N = 1 time; t_link = one NVLink store + flag hop (~2 us, assumed)."""
    if plan.get("kernel") != "lcs16":
        return None
    S, NQ, E = plan["strips"], plan["chunks"], plan["extra_lag"]
    L = 2 * E + 1.9
    t = ms1 / (NQ + 2 * E + (S - 1) * L)
    t_link = 2e-3
    out = {"model": "T(P) = t*(NQ + 2E*P + (S-1)*L) + (P-1)*t_link; weak (n = cols*P): t*(P*NQ + 2E*P + (S-1)*L)",
           "t_chunk_us": round(t * 1e3, 3), "L_chunks": L, "strips": S, "chunks": NQ}
    for P in (1, 2, 4, 8):
        strong = t * (NQ + 2 * E * P + (S - 1) * L) + (P - 1) * t_link
        weak = t * (P * NQ + 2 * E * P + (S - 1) * L) + (P - 1) * t_link
        out[f"P{P}"] = {"strong_ms": round(strong, 3), "strong_speedup": round(ms1 / strong, 3),
                        "weak_ms": round(weak, 3), "weak_efficiency": round(ms1 / weak, 3)}
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
        for name in ("C1", "C2", "C3", "C4", "C6", "C7", "C8"):
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
        if world == 1:
            line["scaling_model"] = scaling_model(head["ms_per_step"], head["plan"], cfg["cols"])
        print(json.dumps(line), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
