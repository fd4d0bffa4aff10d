"""GPU tests of the C-ABI entry points beyond lddp_fill: the host-buffer path (lddp_fill_host,
used by bench.py's e2e leg), empty shapes, argument errors, and the plan's own workspace."""
import ctypes

import numpy as np
import pytest

import oracle
from paper_conf_ipps_kumark15_b200 import inputs

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def L():
    from paper_conf_ipps_kumark15_b200 import lddp
    return lddp


def _host_fill(L, func, category, outputs, a=None, b=None, grid=None, table_shape=None,
               cell=np.int32, table_pitch=None):
    rows, cols = (len(a), len(b)) if grid is None else grid.shape
    d = L.lddp_desc(rows=rows, cols=cols, category=L.CATEGORIES[category], func=L.FUNCS[func],
                    outputs=outputs, param_c=1)
    plan = L.lddp_plan(d)
    try:
        score = np.full(1, -7, cell)
        last_row = np.full(max(cols, 1), -7, cell)
        last_col = np.full(max(rows, 1), -7, cell)
        tbl_full = None if table_shape is None else np.zeros((table_shape[0], table_pitch or table_shape[1]), np.uint8)
        table = None if tbl_full is None else tbl_full[:, :table_shape[1]]
        ptr = lambda x: None if x is None else x.ctypes.data
        inp = L.lddp_inputs(a=ptr(a), b=ptr(b), grid=ptr(grid),
                            grid_pitch=0 if grid is None else grid.strides[0] // grid.itemsize)
        out = L.lddp_outputs(score=ptr(score), last_row=ptr(last_row), last_col=ptr(last_col),
                             table=ptr(tbl_full), table_pitch=0 if table is None else tbl_full.shape[1])
        for _ in range(3):   # repeated calls reuse the plan's staging buffers and workspace
            L.lddp_fill_host(plan, inp, out, 0)
        return score[0], last_row[:cols], last_col[:rows], table
    finally:
        L.lddp_plan_destroy(plan)


def test_fill_host_lcs_dtw(L):
    a, b = inputs.gen_strings(3, 2000, 1700)
    ref = oracle.lcs(a, b)
    s, lr, lc, _ = _host_fill(L, "lcs", "anti_diagonal", L.OUT_SCORE | L.OUT_LAST_ROW | L.OUT_LAST_COL, a=a, b=b)
    assert s == ref.score
    np.testing.assert_array_equal(lr, ref.last_row)
    np.testing.assert_array_equal(lc, ref.last_col)
    x, y = inputs.gen_walks(3, 900, 1300)
    ref = oracle.dtw(x, y)
    s, lr, _, _ = _host_fill(L, "dtw", "anti_diagonal", L.OUT_SCORE | L.OUT_LAST_ROW, a=x, b=y, cell=np.float32)
    assert s.tobytes() == ref.score.tobytes()
    np.testing.assert_array_equal(lr.view(np.int32), ref.last_row.view(np.int32))


def test_fill_host_fs_and_minpath(L):
    img = inputs.gen_image(4, 300, 400, "ramp")
    *_, out = _host_fill(L, "fs", "knight_move", L.OUT_TABLE, grid=img, table_shape=img.shape)
    np.testing.assert_array_equal(out, oracle.fs(img))
    c = inputs.gen_costs(4, 300, 500)
    ref = oracle.minpath3(c)
    s, lr, _, _ = _host_fill(L, "minpath3", "prev_row", L.OUT_SCORE | L.OUT_LAST_ROW, grid=c)
    assert s == ref.score
    np.testing.assert_array_equal(lr, ref.last_row)


@pytest.mark.parametrize("H,W,gpitch,tpitch", [(300, 401, 401, 401), (257, 333, 340, 335), (100, 64, 71, 64),
                                                 (129, 96, 96, 99)])
def test_fill_host_fs_odd_pitches(L, H, W, gpitch, tpitch):
    """Host images and output tables with any pitch (odd widths, pitches not multiples of 4 or 16):
    lddp_fill_host re-pitches its device staging rows, so the word-wide / 16-byte FS paths never
    see a misaligned row."""
    full = inputs.gen_image(H + W, H, gpitch, "uniform")
    img = full[:, :W]
    *_, out = _host_fill(L, "fs", "knight_move", L.OUT_TABLE, grid=img, table_shape=(H, W), table_pitch=tpitch)
    np.testing.assert_array_equal(out, oracle.fs(np.ascontiguousarray(img)))
    c = inputs.gen_costs(H, H, gpitch)[:, :W]
    ref = oracle.minpath3(np.ascontiguousarray(c))
    s, lr, _, _ = _host_fill(L, "minpath3", "prev_row", L.OUT_SCORE | L.OUT_LAST_ROW, grid=c)
    assert s == ref.score
    np.testing.assert_array_equal(lr, ref.last_row)


@pytest.mark.parametrize("m,n", [(0, 0), (0, 5), (5, 0)])
def test_empty_sequences(L, m, n):
    a, b = inputs.gen_strings(1, m, n)
    s, *_ = _host_fill(L, "lcs", "anti_diagonal", L.OUT_SCORE, a=a if m else np.zeros(1, np.uint8)[:0],
                       b=b if n else np.zeros(1, np.uint8)[:0])
    assert s == 0
    s, *_ = _host_fill(L, "levenshtein", "anti_diagonal", L.OUT_SCORE, a=a, b=b)
    assert s == max(m, n)
    x, y = inputs.gen_walks(1, m, n)
    s, *_ = _host_fill(L, "dtw", "anti_diagonal", L.OUT_SCORE, a=x, b=y, cell=np.float32)
    assert (s == 0.0) if (m == 0 and n == 0) else np.isinf(s)


def test_argument_errors(L):
    import torch
    d = L.lddp_desc(rows=100, cols=100, category=L.CAT_ANTI_DIAGONAL, func=L.F_LCS,
                    outputs=L.OUT_SCORE | L.OUT_LAST_ROW)
    plan = L.lddp_plan(d)
    try:
        a = torch.zeros(100, dtype=torch.uint8, device="cuda")
        score = torch.zeros(1, dtype=torch.int32, device="cuda")
        inp = L.lddp_inputs(a=a.data_ptr(), b=a.data_ptr())
        out = L.lddp_outputs(score=score.data_ptr())          # LAST_ROW requested, buffer missing
        with pytest.raises(L.LddpError) as e:
            L.lddp_fill(plan, inp, out, None, 0)
        assert e.value.status == L.LDDP_ERR_INVALID_ARG
        inp = L.lddp_inputs(a=None, b=a.data_ptr())
        out = L.lddp_outputs(score=score.data_ptr(), last_row=score.data_ptr())
        with pytest.raises(L.LddpError) as e:
            L.lddp_fill(plan, inp, out, None, 0)
        assert e.value.status == L.LDDP_ERR_INVALID_ARG
    finally:
        L.lddp_plan_destroy(plan)
    with pytest.raises(L.LddpError) as e:   # FS needs the output image
        L.lddp_plan(L.lddp_desc(rows=10, cols=10, category=L.CAT_KNIGHT_MOVE, func=L.F_FS_DITHER,
                                outputs=L.OUT_SCORE))
    assert e.value.status == L.LDDP_ERR_INVALID_ARG


def test_plan_describe_and_workspace(L):
    d = L.lddp_desc(rows=5000, cols=3000, category=L.CAT_ANTI_DIAGONAL, func=L.F_LCS, outputs=L.OUT_SCORE)
    plan = L.lddp_plan(d)
    try:
        import json
        info = json.loads(L.lddp_plan_describe(plan))
        # LCS without TABLE output runs the packed 16x2 kernel: 64 virtual lanes x P row pairs
        assert info["kernel"] == "lcs16" and info["strips"] >= 1
        assert info["strip_rows"] == 64 * info["rows_per_lane"]
        assert L.lddp_plan_workspace_size(plan) > 0
    finally:
        L.lddp_plan_destroy(plan)
    d = L.lddp_desc(rows=5000, cols=3000, category=L.CAT_ANTI_DIAGONAL, func=L.F_LEVENSHTEIN, outputs=L.OUT_SCORE)
    plan = L.lddp_plan(d)
    try:
        import json
        info = json.loads(L.lddp_plan_describe(plan))
        # the other sequence f's run the 32-bit lane-systolic adiag kernel
        assert info["kernel"] == "adiag" and info["strips"] >= 1
        assert info["strip_rows"] == 32 * info["warps"] * info["rows_per_lane"]
    finally:
        L.lddp_plan_destroy(plan)
    d = L.lddp_desc(rows=500, cols=300, category=L.CAT_ANTI_DIAGONAL, func=L.F_LCS,
                    outputs=L.OUT_SCORE | L.OUT_TABLE)
    plan = L.lddp_plan(d)
    try:
        import json
        # TABLE output: the adiag kernel's staging-tile instantiation (one-warp strips)
        info = json.loads(L.lddp_plan_describe(plan))
        assert info["kernel"] == "adiag" and info["warps"] == 1, info
    finally:
        L.lddp_plan_destroy(plan)
