"""The BASELINE.json workloads C1-C5 and the two synthetic-f
workloads of SURVEY §8(d) "(iL)" / [L298] (C6 inverted-L diagonal max-plus, C7 horizontal
min2-plus) and C8 (batched FS, §8(f)#3): shapes, f, category and the seeded input recipe.  Shared by bench.py,
tools/make_bench_refs.py and the full-size tests."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)
from paper_conf_ipps_kumark15_b200 import inputs  # noqa: E402


def _lcs(n):
    def make(seed):
        a, b = inputs.gen_strings(seed, n, n)
        return {"a": a, "b": b}
    return make


def _dtw(n):
    def make(seed):
        x, y = inputs.gen_walks(seed, n, n)
        return {"a": x, "b": y}
    return make


def _fs(n):
    def make(seed):
        return {"grid": inputs.gen_image(seed, n, n, "ramp")}
    return make


def _fs_batch(n, B):
    def make(seed):
        import numpy as np
        return {"grid": np.concatenate([inputs.gen_image(seed + b, n, n, "ramp") for b in range(B)], axis=0)}
    return make


def _minpath(n):
    def make(seed):
        return {"grid": inputs.gen_costs(seed, n, n)}
    return make


def _init(n):
    def make(seed):
        return {"grid": inputs.gen_init(seed, n, n)}
    return make


CONFIGS = {
    "C1": {"func": "lcs", "category": "anti_diagonal", "rows": 1024, "cols": 1024, "make": _lcs(1024),
           "desc": "LCS of two random 1024-char strings over a 4-letter alphabet (anti-diagonal, int32)"},
    "C2": {"func": "dtw", "category": "anti_diagonal", "rows": 16384, "cols": 16384, "make": _dtw(16384),
           "desc": "DTW of two 16384-sample fp32 random-walk series (anti-diagonal, |x-y| min-plus)"},
    "C3": {"func": "fs", "category": "knight_move", "rows": 8192, "cols": 8192, "make": _fs(8192),
           "desc": "Floyd-Steinberg dithering of a synthetic 8192x8192 grayscale image (knight-move)"},
    "C4": {"func": "minpath3", "category": "prev_row", "rows": 32768, "cols": 32768, "make": _minpath(32768),
           "desc": "previous-row-only 3-neighbour min-path DP on a 32768x32768 random int32 cost grid"},
    "C5": {"func": "lcs", "category": "anti_diagonal", "rows": 100000, "cols": 100000, "make": _lcs(100000),
           "desc": "LCS of two random 100000-char strings, column-strip wavefront pipeline across 1/2/4/8 B200"},
    "C6": {"func": "diagmaxplus", "category": "inverted_l", "rows": 32768, "cols": 32768, "make": _init(32768),
           "param_c": 1,
           "desc": "inverted-L synthetic f = max(init, UL) + 1 [L298] on a 32768x32768 int32 grid (SURVEY 8(d) iL)"},
    "C8": {"func": "fs", "category": "knight_move", "rows": 8 * 8192, "cols": 8192, "batch": 8, "img_rows": 8192,
           "make": _fs_batch(8192, 8),
           "desc": "batched FS: 8 independent 8192x8192 images (seeds 0..7, C3's recipe) in one launch, "
                   "image-parallel (SURVEY 8(f)#3, R21); rows = the stacked batch"},
    "C7": {"func": "min2plus", "category": "prev_row", "rows": 32768, "cols": 32768, "make": _init(32768),
           "param_c": 1,
           "desc": "horizontal case-1 synthetic f = min(UL, U) + 1 [L298] (H1) on a 32768x32768 int32 grid"},
}
