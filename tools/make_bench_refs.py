"""Write tests/golden/bench_refs.json: oracle results for the BASELINE.json configs C1-C5 at
full size (seed 0), used by bench.py and the full-size GPU parity tests.

Calls ONLY oracle/ (and the seeded input generators).  Run: python tools/make_bench_refs.py
C5 (LCS 100000 x 100000, 1e10 cells) takes ~40 s single-threaded."""
import hashlib
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
from paper_conf_ipps_kumark15_b200 import inputs  # noqa: E402

sys.path.insert(0, os.path.join(ROOT, "tools"))
from configs import CONFIGS  # noqa: E402


def digest(arr):
    return hashlib.sha256(np.ascontiguousarray(arr).tobytes()).hexdigest()


def main():
    path = os.path.join(ROOT, "tests", "golden", "bench_refs.json")
    only = sys.argv[1:]   # optional config names: recompute only those, keep the others
    out = {"source": "written by tools/make_bench_refs.py, which calls only oracle/ on the seeded "
                     "inputs of paper_conf_ipps_kumark15_b200/inputs.py (seed 0)", "configs": {}}
    if only and os.path.exists(path):
        with open(path) as f:
            out["configs"] = json.load(f)["configs"]
    for name, cfg in CONFIGS.items():
        if only and name not in only:
            continue
        t0 = time.time()
        x = cfg["make"](0)
        if cfg["func"] in ("lcs", "dtw"):
            r = getattr(oracle, cfg["func"])(x["a"], x["b"])
            score = float(r.score) if cfg["func"] == "dtw" else int(r.score)
            ent = {"score": score, "last_row_sha256": digest(r.last_row), "last_col_sha256": digest(r.last_col)}
        elif cfg["func"] == "fs":
            ir = cfg.get("img_rows", cfg["rows"])   # batched FS: each image of the stack on its own
            g = x["grid"]
            img = np.concatenate([oracle.fs(g[k:k + ir]) for k in range(0, g.shape[0], ir)], axis=0)
            ent = {"image_sha256": digest(img), "white_fraction": float((img == 255).mean())}
        elif cfg["func"] == "minpath3":
            r = oracle.minpath3(x["grid"])
            ent = {"score": int(r.score), "last_row_sha256": digest(r.last_row)}
        elif cfg["func"] == "min2plus":
            r = oracle.min2plus(x["grid"], cfg["param_c"])
            ent = {"score": int(r.score), "last_row_sha256": digest(r.last_row)}
        elif cfg["func"] == "diagmaxplus":
            r = oracle.diagmaxplus(x["grid"], cfg["param_c"])
            ent = {"last_row_sha256": digest(r.last_row), "last_col_sha256": digest(r.last_col)}
        else:
            raise ValueError(cfg["func"])
        ent["oracle_seconds"] = round(time.time() - t0, 2)
        out["configs"][name] = ent
        print(name, ent, flush=True)
    with open(path, "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
