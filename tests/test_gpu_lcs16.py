"""GPU parity of the packed 16x2 LCS kernel (lcs16.cu) against the CPU oracle,
bit-exact: every compiled (P row pairs, E lane lag) geometry on shapes around the strip height
(64P rows, bottom-aligned with virtual rows above row 0), the chunk width (32 columns) and the
band-B lag (32E columns); both match paths (<= 4 distinct characters per warp: PRMT tables;
otherwise the per-warp match table); long fills where the relative values are rebased many times
(LCS up to tens of thousands); grids smaller than the strip count; repeated fills."""
import os

import numpy as np
import pytest

import oracle
from gpu_util import run_gpu
from paper_conf_ipps_kumark15_b200 import inputs

pytestmark = pytest.mark.gpu

GEOMS = [(2, 3), (4, 2), (6, 2), (6, 3), (8, 2)]


def _run(P, E, a, b, **kw):
    old = {k: os.environ.get(k) for k in ("LDDP_L16_P", "LDDP_L16_E")}
    os.environ["LDDP_L16_P"] = str(P)
    os.environ["LDDP_L16_E"] = str(E)
    try:
        got = run_gpu("lcs", "anti_diagonal", a=a, b=b, outputs=("score", "last_row", "last_col"), **kw)
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v
    plan = got["plan"]
    assert '"lcs16"' in plan and f'"rows_per_lane": {P},' in plan and f'"extra_lag": {E},' in plan, plan
    return got


def _check(got, ref):
    assert int(got["score"]) == int(ref.score)
    np.testing.assert_array_equal(got["last_row"], ref.last_row, err_msg="last_row")
    np.testing.assert_array_equal(got["last_col"], ref.last_col, err_msg="last_col")


def _cases():
    for P, E in GEOMS:
        sh = 64 * P
        for m, n in [(1, 1), (1, 70), (70, 1), (sh - 1, 33), (sh, 32), (sh + 1, 31), (2 * sh + 5, 41),
                     (3 * sh - 7, 72), (sh // 2 + 3, 1000), (997, 1009), (sh + 3, 32 * E - 1), (sh, 64 * E + 1),
                     (5, 2 * 32 * E + 33)]:
            yield P, E, m, n


@pytest.mark.parametrize("P,E,m,n", list(_cases()))
def test_lcs16_geometry(P, E, m, n):
    a, b = inputs.gen_strings(17 * m + n + P, m, n)
    _check(_run(P, E, a, b), oracle.lcs(a, b))


@pytest.mark.parametrize("P,E", GEOMS)
@pytest.mark.parametrize("alphabet", ["bytes", "mixed", "ascii26", "one", "two"])
def test_lcs16_alphabets(P, E, alphabet):
    """<= 4 distinct row characters per warp take the PRMT tables, others the match table; 'mixed'
    puts warps of both kinds in one fill; 'one' (a single letter: LCS grows one per column, the
    largest relative range) and 'two' stress the rebase."""
    m, n = 1500, 2300
    rng = np.random.default_rng(m + 7 * n + P + 10 * E)
    if alphabet == "bytes":
        a = rng.integers(0, 256, m, dtype=np.uint8)
        b = rng.integers(0, 256, n, dtype=np.uint8)
    elif alphabet == "ascii26":
        a = rng.integers(65, 91, m).astype(np.uint8)
        b = rng.integers(65, 91, n).astype(np.uint8)
    elif alphabet == "one":
        a = np.full(m, 65, np.uint8)
        b = np.full(n, 65, np.uint8)
    elif alphabet == "two":
        a = rng.integers(0, 2, m).astype(np.uint8) + 48
        b = rng.integers(0, 2, n).astype(np.uint8) + 48
    else:
        a = np.concatenate([np.frombuffer(b"ACGT", np.uint8)[rng.integers(0, 4, m // 2)],
                            rng.integers(60, 80, m - m // 2).astype(np.uint8)])
        b = np.concatenate([np.frombuffer(b"ACGT", np.uint8)[rng.integers(0, 4, n // 2)],
                            rng.integers(0, 256, n - n // 2).astype(np.uint8)])
    _check(_run(P, E, a, b), oracle.lcs(a, b))


@pytest.mark.parametrize("m,n,alphabet", [(20000, 30001, "dna"), (3000, 70003, "one"), (70001, 2500, "one"),
                                          (9000, 9000, "bytes")])
def test_lcs16_long(m, n, alphabet):
    """Values far beyond 16 bits (rebased many times); the planner's default geometry."""
    rng = np.random.default_rng(m ^ n)
    if alphabet == "dna":
        a, b = inputs.gen_strings(m + n, m, n)
    elif alphabet == "one":
        a, b = np.full(m, 67, np.uint8), np.full(n, 67, np.uint8)
    else:
        a = rng.integers(0, 256, m, dtype=np.uint8)
        b = rng.integers(0, 256, n, dtype=np.uint8)
    got = run_gpu("lcs", "anti_diagonal", a=a, b=b, outputs=("score", "last_row", "last_col"))
    assert '"lcs16"' in got["plan"]
    _check(got, oracle.lcs(a, b))


@pytest.mark.parametrize("grid", [1, 2, 5])
def test_lcs16_small_grid(grid):
    """More strips than CTAs: each CTA runs several strips in claim order; several fills reuse
    one workspace (epoch-tagged boundary pairs)."""
    m, n = 192 * 7 + 17, 777
    a, b = inputs.gen_strings(grid, m, n)
    _check(_run(2, 3, a, b, grid_ctas=grid, reps=3), oracle.lcs(a, b))


@pytest.mark.parametrize("P,E", GEOMS)
@pytest.mark.parametrize("alphabet", ["one", "dna"])
def test_lcs16_rebase_every_geometry(P, E, alphabet):
    """Values far above the rebase threshold (8192) in every compiled geometry: the relative
    16-bit encoding is rebased many times per strip, with the widest value spread the geometry
    allows (one letter: LCS grows by one per column and row)."""
    m, n = (12001, 13003) if alphabet == "one" else (14000, 15001)
    if alphabet == "one":
        a, b = np.full(m, 71, np.uint8), np.full(n, 71, np.uint8)
    else:
        a, b = inputs.gen_strings(P * 10 + E, m, n)
    _check(_run(P, E, a, b), oracle.lcs(a, b))
