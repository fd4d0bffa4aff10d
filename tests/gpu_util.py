"""Helpers for the GPU parity tests: run one fill through the C ABI (liblddp.so via the ctypes
binding) on numpy inputs and return numpy outputs.  No arithmetic of the method here."""
import numpy as np

SEQ_FUNCS = ("lcs", "levenshtein", "dtw")
OUT_DTYPE = {"lcs": np.int32, "levenshtein": np.int32, "dtw": np.float32, "fs": np.uint8,
             "minpath3": np.int32, "min2plus": np.int32, "diagmaxplus": np.int32}


def run_gpu(func, category, *, a=None, b=None, grid=None, outputs=("score", "last_row"),
            param_c=1, tile_rows=0, grid_ctas=0, table_pad=0, reps=1, grid_pad=0, band_rows=0):
    import torch

    from paper_conf_ipps_kumark15_b200 import lddp

    dev = torch.device("cuda:0")
    if func in SEQ_FUNCS:
        rows, cols = len(a), len(b)
    else:
        rows, cols = grid.shape
    bits = 0
    names = {"score": lddp.OUT_SCORE, "last_row": lddp.OUT_LAST_ROW, "last_col": lddp.OUT_LAST_COL,
             "table": lddp.OUT_TABLE}
    for o in outputs:
        bits |= names[o]
    plan = lddp.Plan(func, category, rows, cols, bits, param_c=param_c, tile_rows=tile_rows,
                     grid_ctas=grid_ctas, band_rows=band_rows)
    vdt = {np.int32: torch.int32, np.float32: torch.float32}
    cell_dt = torch.float32 if func == "dtw" else torch.int32
    t = {}
    if func in SEQ_FUNCS:
        t["a"] = torch.from_numpy(np.ascontiguousarray(a)).to(dev)
        t["b"] = torch.from_numpy(np.ascontiguousarray(b)).to(dev)
    else:
        g = np.ascontiguousarray(grid)
        if (func == "fs" and cols % 4) or grid_pad:
            pad = np.zeros((rows, cols + (-cols) % 4 + grid_pad), g.dtype)   # row pitch > cols
            pad[:, :cols] = g
            t["grid"] = torch.from_numpy(pad).to(dev)[:, :cols]
        else:
            t["grid"] = torch.from_numpy(g).to(dev)
    res = {}
    if "score" in outputs:
        t["score"] = torch.full((1,), -7, dtype=cell_dt, device=dev)
    if "last_row" in outputs:
        t["last_row"] = torch.full((max(cols, 1),), -7, dtype=cell_dt, device=dev)
    if "last_col" in outputs:
        t["last_col"] = torch.full((max(rows, 1),), -7, dtype=cell_dt, device=dev)
    if "table" in outputs:
        tdt = torch.uint8 if func == "fs" else cell_dt
        pitch = cols + table_pad
        if func == "fs":
            pitch += (-pitch) % 4
        t["table"] = torch.full((max(rows, 1), max(pitch, 1)), 7, dtype=tdt, device=dev)
    for _ in range(reps):
        plan.fill(**t)
    plan.check()
    torch.cuda.synchronize()
    if "score" in outputs:
        res["score"] = t["score"].cpu().numpy()[0]
    if "last_row" in outputs:
        res["last_row"] = t["last_row"].cpu().numpy()[:cols]
    if "last_col" in outputs:
        res["last_col"] = t["last_col"].cpu().numpy()[:rows]
    if "table" in outputs:
        res["table"] = t["table"].cpu().numpy()[:rows, :cols]
    res["plan"] = plan.info
    return res
