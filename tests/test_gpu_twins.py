"""GPU parity of the two symmetric twins of Table I [L109-L113] ("Vertical is the transpose of
Horizontal, mInverted-L the mirror of Inverted-L" [L111], reading R15) against the CPU oracle,
bit-exact: MIN2_PLUS_V in the VERTICAL category (tiled transpose into the workspace + the
prev-row plan of the transposed problem) and ANTIDIAG_MAXPLUS in the MINVERTED_L category (the
inverted-L kernel reading the grid mirrored).  Score / last column / last row / full table, odd
shapes, row pitches wider than the grid, the host-buffer path."""
import numpy as np
import pytest

import oracle
from gpu_util import run_gpu
from paper_conf_ipps_kumark15_b200 import inputs

pytestmark = pytest.mark.gpu

SHAPES = [(1, 1), (1, 57), (63, 1), (100, 300), (333, 77), (1000, 1203), (2048, 64), (97, 4099)]


@pytest.mark.parametrize("H,W", SHAPES)
@pytest.mark.parametrize("c", [0, 1, 3])
def test_vertical_min2plus_v(H, W, c):
    init = inputs.gen_init(H * 7 + W + c, H, W)
    ref = oracle.min2plus_v(init, c, table=True)
    got = run_gpu("min2plus_v", "vertical", grid=init, outputs=("score", "last_col", "table"), param_c=c)
    assert '"transpose+prevrow"' in got["plan"]
    assert got["score"] == ref.score
    np.testing.assert_array_equal(got["last_col"], ref.last_col)
    np.testing.assert_array_equal(got["table"], ref.table)
    got = run_gpu("min2plus_v", "vertical", grid=init, outputs=("score", "last_col"), param_c=c, reps=2)
    assert got["score"] == ref.score
    np.testing.assert_array_equal(got["last_col"], ref.last_col)


@pytest.mark.parametrize("H,W", SHAPES)
@pytest.mark.parametrize("c", [0, 1, 2])
def test_minverted_l_antidiag_maxplus(H, W, c):
    init = inputs.gen_init(H * 5 + W + c, H, W)
    ref = oracle.antidiag_maxplus(init, c, table=True)
    got = run_gpu("antidiag_maxplus", "minverted_l", grid=init, outputs=("last_row", "last_col", "table"),
                  param_c=c, table_pad=5)
    assert '"invl"' in got["plan"] and '"mirror": 1' in got["plan"]
    np.testing.assert_array_equal(got["last_row"], ref.last_row)
    np.testing.assert_array_equal(got["last_col"], ref.last_col)   # column 0: where the chains end
    np.testing.assert_array_equal(got["table"], ref.table)


def test_twins_pitched_grids():
    """Grids whose row pitch exceeds their width (a column slice of a wider array)."""
    init = inputs.gen_init(3, 500, 613)
    ref = oracle.min2plus_v(init, 2, table=True)
    got = run_gpu("min2plus_v", "vertical", grid=init, outputs=("score", "last_col", "table"), param_c=2,
                  grid_pad=87)
    assert got["score"] == ref.score
    np.testing.assert_array_equal(got["table"], ref.table)
    ref = oracle.antidiag_maxplus(init, 2, table=True)
    got = run_gpu("antidiag_maxplus", "minverted_l", grid=init, outputs=("last_row", "last_col", "table"), param_c=2,
                  grid_pad=87)
    np.testing.assert_array_equal(got["table"], ref.table)
    np.testing.assert_array_equal(got["last_col"], ref.last_col)
