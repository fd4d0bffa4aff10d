"""GPU parity of the column-block persistent prev-row kernel (csrc/prevrow_cb.cu) against the
CPU oracle, bit-exact: every compiled geometry (VP, HB, D) and warps-per-CTA setting, shapes
spanning several bands (HB rows) and column blocks with ragged last band / block, W % 4 == 0
(the kernel's precondition; other widths take the fallback kernel, covered in
test_gpu_parity.py), repeated fills on one workspace (epoch-tagged edge pairs)."""
import json
import os

import numpy as np
import pytest

import oracle
from gpu_util import run_gpu
from paper_conf_ipps_kumark15_b200 import inputs

pytestmark = pytest.mark.gpu

CB_SHAPES = [(1, 4), (2, 8), (63, 132), (64, 256), (65, 260), (129, 388), (1000, 1000),
             (777, 2052), (130, 4096), (3001, 516), (4100, 8196)]


@pytest.fixture
def cb_env():
    keys = ("LDDP_CB_VARIANT", "LDDP_CB_WARPS", "LDDP_HX_VARIANT")
    old = {k: os.environ.get(k) for k in keys}

    def set_(variant, warps):
        os.environ["LDDP_CB_VARIANT"] = str(variant)
        os.environ["LDDP_CB_WARPS"] = str(warps)
        os.environ["LDDP_HX_VARIANT"] = "-1"   # SCORE / LAST_ROW fills would take prevrow_hx

    yield set_
    for k, v in old.items():
        if v is None:
            os.environ.pop(k, None)
        else:
            os.environ[k] = v


@pytest.mark.parametrize("variant,warps", [(0, 2), (0, 1), (0, 4), (5, 4), (5, 2), (5, 1), (13, 2), (13, 4), (13, 8), (17, 4), (17, 2)])
@pytest.mark.parametrize("shape", CB_SHAPES)
def test_minpath3_cb(cb_env, variant, warps, shape):
    cb_env(variant, warps)
    H, W = shape
    c = inputs.gen_costs(17 * H + W, H, W)
    ref = oracle.minpath3(c, table=(H * W <= 1 << 20))
    outs = ("score", "last_row", "table") if ref.table is not None else ("score", "last_row")
    got = run_gpu("minpath3", "prev_row", grid=c, outputs=outs, reps=2)
    info = json.loads(got["plan"])
    assert info["kernel"] == "prevrow_cb", info
    assert info["variant"] == variant
    np.testing.assert_array_equal(got["last_row"], ref.last_row)
    assert got["score"] == ref.score
    if "table" in outs:
        np.testing.assert_array_equal(got["table"], ref.table)


@pytest.mark.parametrize("variant", [0, 5, 13, 17])
@pytest.mark.parametrize("shape", [(1000, 1000), (300, 2052)])
def test_min2plus_diagmaxplus_cb(cb_env, variant, shape):
    cb_env(variant, 2)
    H, W = shape
    init = inputs.gen_init(H + 3 * W, H, W, hi=10000)
    ref = oracle.min2plus(init, 3, table=True)
    got = run_gpu("min2plus", "prev_row", grid=init, param_c=3, outputs=("score", "last_row", "table"))
    assert json.loads(got["plan"])["kernel"] == "prevrow_cb"
    np.testing.assert_array_equal(got["table"], ref.table)
    assert got["score"] == ref.score
    ref = oracle.diagmaxplus(init, 2, table=True)
    got = run_gpu("diagmaxplus", "prev_row", grid=init, param_c=2, outputs=("last_row", "table"))
    np.testing.assert_array_equal(got["table"], ref.table)
    np.testing.assert_array_equal(got["last_row"], ref.last_row)


def test_cb_disabled_falls_back(cb_env):
    """LDDP_CB_VARIANT=-1 selects the claimed-task kernel; same results."""
    cb_env(-1, 2)
    c = inputs.gen_costs(3, 500, 1000)
    ref = oracle.minpath3(c)
    got = run_gpu("minpath3", "prev_row", grid=c, outputs=("score", "last_row"))
    assert json.loads(got["plan"])["kernel"] == "prevrow"
    assert got["score"] == ref.score
    np.testing.assert_array_equal(got["last_row"], ref.last_row)


@pytest.mark.parametrize("band_rows,variant", [(16, 13), (32, 5), (48, 17), (64, 0)])
@pytest.mark.parametrize("func", ["minpath3", "min2plus"])
def test_band_rows_selects_band_height(band_rows, variant, func):
    """lddp_desc.band_rows = the trapezoid band height HB of the column-block kernel."""
    H, W = 1000, 1536
    g = inputs.gen_costs(band_rows + H, H, W) if func == "minpath3" else inputs.gen_init(band_rows, H, W)
    ref = oracle.minpath3(g) if func == "minpath3" else oracle.min2plus(g, 1)
    got = run_gpu(func, "prev_row", grid=g, outputs=("score", "last_row"), band_rows=band_rows)
    assert f'"kernel": "prevrow_cb", "variant": {variant},' in got["plan"], got["plan"]
    assert got["score"] == ref.score
    np.testing.assert_array_equal(got["last_row"], ref.last_row)


def test_band_rows_unsupported_height():
    from paper_conf_ipps_kumark15_b200 import lddp
    with pytest.raises(lddp.LddpError) as e:
        lddp.Plan("minpath3", "prev_row", 100, 128, lddp.OUT_SCORE, band_rows=40)
    assert e.value.status == lddp.LDDP_ERR_UNSUPPORTED
