"""GPU parity: every (f, covering category, geometry variant) through the C ABI against the CPU
oracle, element by element, on seeded inputs at awkward shapes (1x1, 1xn, nx1, primes, tile
and chunk sizes +-1, ragged strips / bands).  Integer f's and FS must be bit-exact; DTW is
expected bit-exact (same per-cell operation sequence) and is held to <= 1e-5 relative, the north
star's tolerance.  Schedule independence: the same f under every covering category gives the
identical table."""
import json

import numpy as np
import pytest

import oracle
from gpu_util import run_gpu
from paper_conf_ipps_kumark15_b200 import inputs

pytestmark = pytest.mark.gpu

# strip rows of the anti-diagonal kernel = 4 warps x 32 lanes x R  (R = 4 -> 512)
SEQ_SHAPES = [(1, 1), (1, 40), (40, 1), (2, 3), (7, 13), (31, 33), (100, 257), (511, 64),
              (512, 65), (513, 95), (997, 1009), (1300, 200), (129, 1500)]
AD_VARIANTS = [4, 2, 8]       # tile_rows: R4 (chain), R2 (skewed), R8 (skewed)
KN_VARIANTS = [1, 2]


def _seq_inputs(func, seed, m, n):
    if func == "dtw":
        return inputs.gen_walks(seed, m, n)
    return inputs.gen_strings(seed, m, n)


def _oracle_seq(func, a, b, table=False):
    return {"lcs": oracle.lcs, "levenshtein": oracle.levenshtein, "dtw": oracle.dtw}[func](a, b, table=table)


def _assert_close(func, got, ref):
    if func == "dtw":
        got = np.asarray(got, np.float32)
        ref = np.asarray(ref, np.float32)
        assert np.allclose(got, ref, rtol=1e-5, atol=0), (got, ref)
        # expected bit-exact: report if not
        assert np.array_equal(got.view(np.int32), ref.view(np.int32))
    else:
        np.testing.assert_array_equal(got, ref)


@pytest.mark.parametrize("func", ["lcs", "levenshtein", "dtw"])
@pytest.mark.parametrize("shape", SEQ_SHAPES)
def test_seq_table_antidiag(func, shape):
    m, n = shape
    a, b = _seq_inputs(func, 1000 + m * 7 + n, m, n)
    ref = _oracle_seq(func, a, b, table=True)
    got = run_gpu(func, "anti_diagonal", a=a, b=b,
                  outputs=("score", "last_row", "last_col", "table"), table_pad=3)
    _assert_close(func, got["table"], ref.table)
    _assert_close(func, got["last_row"], ref.last_row)
    _assert_close(func, got["last_col"], ref.last_col)
    _assert_close(func, got["score"], ref.score)


@pytest.mark.parametrize("func", ["lcs", "levenshtein", "dtw"])
@pytest.mark.parametrize("rows", AD_VARIANTS)
@pytest.mark.parametrize("shape", [(1, 1), (3, 5), (513, 95), (997, 1009), (2100, 1700), (4097, 333)])
def test_seq_variants_antidiag(func, rows, shape):
    m, n = shape
    a, b = _seq_inputs(func, 7 * m + n + rows, m, n)
    ref = _oracle_seq(func, a, b)
    got = run_gpu(func, "anti_diagonal", a=a, b=b, outputs=("score", "last_row", "last_col"),
                  tile_rows=rows)
    _assert_close(func, got["last_row"], ref.last_row)
    _assert_close(func, got["last_col"], ref.last_col)
    _assert_close(func, got["score"], ref.score)


@pytest.mark.parametrize("func", ["lcs", "levenshtein", "dtw"])
@pytest.mark.parametrize("rows", AD_VARIANTS)
@pytest.mark.parametrize("shape", [(3, 5), (513, 95), (997, 1009), (2100, 1700)])
def test_seq_variants_wavefront_kernel(func, rows, shape, monkeypatch):
    """The strip-wavefront kernel (default for TABLE outputs) on score / last-row / last-column."""
    monkeypatch.setenv("LDDP_KERNEL", "wavefront")
    m, n = shape
    a, b = _seq_inputs(func, 11 * m + n + rows, m, n)
    ref = _oracle_seq(func, a, b)
    got = run_gpu(func, "anti_diagonal", a=a, b=b, outputs=("score", "last_row", "last_col"),
                  tile_rows=rows)
    assert '"wavefront"' in got["plan"]
    _assert_close(func, got["last_row"], ref.last_row)
    _assert_close(func, got["last_col"], ref.last_col)
    _assert_close(func, got["score"], ref.score)


@pytest.mark.parametrize("func", ["lcs", "levenshtein", "dtw"])
@pytest.mark.parametrize("rows", KN_VARIANTS)
@pytest.mark.parametrize("shape", [(1, 1), (5, 2), (300, 257), (1025, 999)])
def test_seq_under_knight_schedule(func, rows, shape):
    """Schedule independence: anti-diagonal f's under the knight-move category."""
    m, n = shape
    a, b = _seq_inputs(func, 3 * m + n, m, n)
    ref = _oracle_seq(func, a, b, table=True)
    got = run_gpu(func, "knight_move", a=a, b=b, outputs=("score", "table", "last_col"), tile_rows=rows)
    _assert_close(func, got["table"], ref.table)
    _assert_close(func, got["last_col"], ref.last_col)
    _assert_close(func, got["score"], ref.score)


FS_SHAPES = [(1, 1), (1, 8), (8, 1), (2, 2), (3, 3), (4, 4), (5, 7), (33, 65), (127, 129),
             (200, 300), (257, 1000), (1031, 517)]


@pytest.mark.parametrize("rows", KN_VARIANTS)
@pytest.mark.parametrize("shape", FS_SHAPES)
@pytest.mark.parametrize("kind", ["ramp", "uniform"])
def test_fs_knight(rows, shape, kind):
    H, W = shape
    img = inputs.gen_image(H * 13 + W, H, W, kind)
    got = run_gpu("fs", "knight_move", grid=img, outputs=("table",), tile_rows=rows)
    np.testing.assert_array_equal(got["table"], oracle.fs(img))


def test_fs_golden_examples():
    from conftest import golden
    for case in golden("fs_examples.json")["cases"]:
        img = np.array(case["in"], np.uint8)
        got = run_gpu("fs", "knight_move", grid=img, outputs=("table",))
        np.testing.assert_array_equal(got["table"], np.array(case["out"], np.uint8), err_msg=case["name"])


GRID_SHAPES = [(1, 1), (1, 300), (300, 1), (2, 2), (31, 127), (32, 128), (33, 129), (64, 256),
               (65, 257), (100, 1000), (257, 383), (1000, 130)]


@pytest.mark.parametrize("category", ["prev_row", "knight_move"])
@pytest.mark.parametrize("shape", GRID_SHAPES)
def test_minpath3(category, shape):
    H, W = shape
    c = inputs.gen_costs(H + 31 * W, H, W)
    ref = oracle.minpath3(c, table=True)
    got = run_gpu("minpath3", category, grid=c, outputs=("score", "last_row", "table"), table_pad=1)
    np.testing.assert_array_equal(got["table"], ref.table)
    np.testing.assert_array_equal(got["last_row"], ref.last_row)
    assert got["score"] == ref.score


@pytest.mark.parametrize("category", ["prev_row", "knight_move", "anti_diagonal"])
@pytest.mark.parametrize("shape", GRID_SHAPES)
def test_min2plus(category, shape):
    H, W = shape
    init = inputs.gen_init(H * 3 + W, H, W, hi=10000)
    ref = oracle.min2plus(init, 3, table=True)
    got = run_gpu("min2plus", category, grid=init, param_c=3, outputs=("score", "last_row", "table"))
    np.testing.assert_array_equal(got["table"], ref.table)
    np.testing.assert_array_equal(got["last_row"], ref.last_row)
    assert got["score"] == ref.score


@pytest.mark.parametrize("category", ["inverted_l", "prev_row", "knight_move", "anti_diagonal"])
@pytest.mark.parametrize("shape", GRID_SHAPES)
def test_diagmaxplus(category, shape):
    H, W = shape
    init = inputs.gen_init(H * 5 + W, H, W)
    ref = oracle.diagmaxplus(init, 2, table=True)
    outs = ("last_row", "table") if category == "prev_row" else ("last_row", "last_col", "table")
    got = run_gpu("diagmaxplus", category, grid=init, param_c=2, outputs=outs)
    np.testing.assert_array_equal(got["table"], ref.table)
    np.testing.assert_array_equal(got["last_row"], ref.last_row)
    if "last_col" in outs:
        np.testing.assert_array_equal(got["last_col"], ref.last_col)


def test_repeated_fills_reuse_workspace():
    """Epoch-tagged flags: many fills on one workspace without re-initialisation."""
    a, b = inputs.gen_strings(5, 1500, 1400)
    ref = oracle.lcs(a, b)
    got = run_gpu("lcs", "anti_diagonal", a=a, b=b, outputs=("score", "last_row"), reps=25)
    assert got["score"] == ref.score
    np.testing.assert_array_equal(got["last_row"], ref.last_row)


def test_small_grid_forces_strip_reuse():
    """A 1-CTA / 2-CTA persistent grid must process every strip in claim order."""
    a, b = inputs.gen_strings(6, 3000, 777)
    ref = oracle.lcs(a, b)
    for g in (1, 2, 3):
        got = run_gpu("lcs", "anti_diagonal", a=a, b=b, outputs=("score", "last_row", "last_col"), grid_ctas=g)
        assert got["score"] == ref.score
        np.testing.assert_array_equal(got["last_row"], ref.last_row)
        np.testing.assert_array_equal(got["last_col"], ref.last_col)
    c = inputs.gen_costs(8, 200, 700)
    r = oracle.minpath3(c)
    got = run_gpu("minpath3", "prev_row", grid=c, outputs=("score", "last_row"), grid_ctas=1)
    assert got["score"] == r.score
    np.testing.assert_array_equal(got["last_row"], r.last_row)


@pytest.mark.parametrize("func", ["lcs", "levenshtein", "dtw"])
@pytest.mark.parametrize("shape", [(1, 1), (1, 300), (300, 1), (127, 33), (128, 64), (129, 95), (385, 1000),
                                   (1000, 777), (2000, 2049)])
@pytest.mark.parametrize("kernel", ["default", "wavefront"])
def test_table_fill_kernels(func, shape, kernel, monkeypatch):
    """TABLE fills of the anti-diagonal sequence f's: the adiag staging-tile kernel (default) and
    the wavefront kernel (LDDP_KERNEL=wavefront) both equal the oracle's table element by element
    (bit-exact for LCS / Levenshtein; DTW too: same fp32 operation order)."""
    if kernel == "wavefront":
        monkeypatch.setenv("LDDP_KERNEL", "wavefront")
    m, n = shape
    if func == "dtw":
        a, b = inputs.gen_walks(7 * m + n, m, n)
        ref = oracle.dtw(a, b, table=True)
    else:
        a, b = inputs.gen_strings(7 * m + n, m, n)
        ref = getattr(oracle, func)(a, b, table=True)
    got = run_gpu(func, "anti_diagonal", a=a, b=b, outputs=("score", "table"))
    assert json.loads(got["plan"])["kernel"] == ("wavefront" if kernel == "wavefront" else "adiag")
    np.testing.assert_array_equal(got["table"], ref.table)
    assert got["score"] == ref.score
