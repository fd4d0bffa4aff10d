"""GPU parity of the lane-systolic anti-diagonal kernel (adiag.cuh) against the CPU oracle:
every compiled (rows per lane R, lane lag E) geometry, shapes around the strip height
(4 warps x 32 lanes x R rows, bottom-aligned with virtual rows above row 0) and the chunk width
(32 columns), persistent grids smaller than the strip count (several strips per CTA), repeated
fills on one workspace (epoch-tagged boundary pairs).  LCS / Levenshtein bit-exact; DTW
bit-exact and <= 1e-5 relative (north star)."""
import os
import sys

import numpy as np
import pytest

import oracle
from gpu_util import run_gpu
from paper_conf_ipps_kumark15_b200 import inputs

pytestmark = pytest.mark.gpu

sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools"))
from gen_adiag import GEOMS as _GEN  # noqa: E402  (the compiled (R, E, W) geometries)

GEOMS = {"lcs": _GEN["LCS"][1], "levenshtein": _GEN["LEVENSHTEIN"][1], "dtw": _GEN["DTW"][1]}


def _inputs(func, seed, m, n):
    if func == "dtw":
        return inputs.gen_walks(seed, m, n)
    return inputs.gen_strings(seed, m, n)


def _ref(func, a, b):
    return {"lcs": oracle.lcs, "levenshtein": oracle.levenshtein, "dtw": oracle.dtw}[func](a, b)


def _check(func, got, ref):
    for k in ("score", "last_row", "last_col"):
        g, r = np.asarray(got[k]), np.asarray(getattr(ref, k))
        if func == "dtw":
            assert np.allclose(g, r, rtol=1e-5, atol=0), k
            assert np.array_equal(g.astype(np.float32).view(np.int32), r.astype(np.float32).view(np.int32)), k
        else:
            np.testing.assert_array_equal(g, r, err_msg=k)


def _run(func, R, E, W, a, b, S=0, **kw):
    old = {k: os.environ.get(k) for k in ("LDDP_AD_E", "LDDP_AD_W", "LDDP_AD_S", "LDDP_KERNEL")}
    os.environ["LDDP_KERNEL"] = "adiag"   # LCS defaults to lcs16.cu (test_gpu_lcs16.py)
    os.environ["LDDP_AD_E"] = str(E)
    os.environ["LDDP_AD_W"] = str(W)
    os.environ["LDDP_AD_S"] = str(S)
    try:
        got = run_gpu(func, "anti_diagonal", a=a, b=b, outputs=("score", "last_row", "last_col"),
                      tile_rows=R, **kw)
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v
    plan = got["plan"]
    assert '"adiag"' in plan and f'"rows_per_lane": {R},' in plan and f'"extra_lag": {E},' in plan, plan
    assert f'"warps": {W},' in plan and f'"skew": {S},' in plan, plan
    return got


def _cases():
    for func, geoms in GEOMS.items():
        for geom in geoms:
            R, E, W = geom[:3]
            S = geom[3] if len(geom) > 3 else 0   # split: lower half of the rows one column behind
            sh = 32 * W * R
            for m, n in [(1, 1), (1, 70), (70, 1), (sh - 1, 33), (sh, 32), (sh + 1, 31), (2 * sh + 5, 41),
                         (3 * sh - 7, 72), (sh // 2 + 3, 1000), (997, 1009)]:
                yield func, R, E, W, S, m, n


@pytest.mark.parametrize("func,R,E,W,S,m,n", list(_cases()))
def test_adiag_geometry(func, R, E, W, S, m, n):
    a, b = _inputs(func, 31 * m + n + R, m, n)
    _check(func, _run(func, R, E, W, a, b, S=S), _ref(func, a, b))


@pytest.mark.parametrize("func", ["lcs", "levenshtein", "dtw"])
@pytest.mark.parametrize("grid", [1, 2, 3])
def test_adiag_small_grid(func, grid):
    """More strips than CTAs: each CTA runs several strips in claim order (deadlock-free)."""
    R, E, W = GEOMS[func][0][:3]
    m, n = 32 * W * R * 5 + 17, 300
    a, b = _inputs(func, 5 + grid, m, n)
    _check(func, _run(func, R, E, W, a, b, grid_ctas=grid, reps=3), _ref(func, a, b))


@pytest.mark.parametrize("func", ["lcs", "levenshtein", "dtw"])
def test_adiag_large(func):
    """A few thousand rows and columns with the planner's own geometry choice."""
    m, n = 6001, 5003
    a, b = _inputs(func, 77, m, n)
    got = run_gpu(func, "anti_diagonal", a=a, b=b, outputs=("score", "last_row", "last_col"), reps=2)
    assert ('"lcs16"' if func == "lcs" else '"adiag"') in got["plan"]
    _check(func, got, _ref(func, a, b))


@pytest.mark.parametrize("func", ["lcs", "levenshtein"])
@pytest.mark.parametrize("alphabet", ["bytes", "mixed", "ascii26"])
@pytest.mark.parametrize("shape", [(700, 900), (3001, 517)])
def test_adiag_alphabets(func, alphabet, shape):
    """Match cells take two paths per warp: <= 4 distinct row characters (DNA: a per-lane packed
    mask register, one PRMT per step) or the per-warp 256-entry match table.  Cover both and warps
    of both kinds in one fill."""
    m, n = shape
    rng = np.random.default_rng(m + 3 * n)
    if alphabet == "bytes":
        a = rng.integers(0, 256, m, dtype=np.uint8)
        b = rng.integers(0, 256, n, dtype=np.uint8)
    elif alphabet == "ascii26":
        a = rng.integers(65, 91, m).astype(np.uint8)
        b = rng.integers(65, 91, n).astype(np.uint8)
    else:   # first half DNA (small-alphabet warps), second half wide (table warps)
        a = np.concatenate([np.frombuffer(b"ACGT", np.uint8)[rng.integers(0, 4, m // 2)],
                            rng.integers(60, 80, m - m // 2).astype(np.uint8)])
        b = np.concatenate([np.frombuffer(b"ACGT", np.uint8)[rng.integers(0, 4, n // 2)],
                            rng.integers(60, 80, n - n // 2).astype(np.uint8)])
    got = run_gpu(func, "anti_diagonal", a=a, b=b, outputs=("score", "last_row", "last_col"))
    _check(func, got, _ref(func, a, b))
