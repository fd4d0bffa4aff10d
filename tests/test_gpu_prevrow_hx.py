"""GPU parity of the hierarchical-exchange prev-row kernel (csrc/prevrow_hx.cu) against the CPU
oracle, bit-exact: every compiled geometry (NW, HBI, HBO, D, GH), shapes spanning several CTAs
(CW columns), inner bands (HBI rows), outer bands (HBO rows) and ring wraps (D rows), with
ragged last band / period / CTA, tables narrower than one CTA or one warp, W % 4 == 0 (the
kernel's precondition), every prev-row f compiled for it, repeated fills on one workspace
(epoch-tagged outer edge pairs), and the dispatch rules (TABLE and band_rows keep prevrow_cb)."""
import json
import os

import numpy as np
import pytest

import oracle
from gpu_util import run_gpu
from paper_conf_ipps_kumark15_b200 import inputs

pytestmark = pytest.mark.gpu

VARIANTS = [0, 2, 6, 8]
CTA_COLS = {0: 224, 2: 224, 6: 288, 8: 224}   # own columns per CTA (one CTA per SM)
HX_SHAPES = [(1, 4), (2, 8), (3, 12), (17, 132), (64, 256), (97, 224), (96, 448), (193, 452),
             (1000, 1000), (777, 2052), (130, 4096), (3001, 516), (4100, 8196), (257, 32768)]


@pytest.fixture
def hx_env():
    old = os.environ.get("LDDP_HX_VARIANT")

    def set_(variant):
        os.environ["LDDP_HX_VARIANT"] = str(variant)

    yield set_
    if old is None:
        os.environ.pop("LDDP_HX_VARIANT", None)
    else:
        os.environ["LDDP_HX_VARIANT"] = old


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("shape", HX_SHAPES)
def test_minpath3_hx(hx_env, variant, shape):
    hx_env(variant)
    H, W = shape
    if -(-W // CTA_COLS[variant]) > 148:
        pytest.skip("more CTAs than SMs: the plan keeps prevrow_cb")
    c = inputs.gen_costs(31 * H + W, H, W)
    tab = H * W <= 1 << 20
    ref = oracle.minpath3(c, table=tab)
    outs = ("score", "last_row", "table") if tab else ("score", "last_row")
    got = run_gpu("minpath3", "prev_row", grid=c, outputs=outs, reps=2)
    info = json.loads(got["plan"])
    assert info["kernel"] == "prevrow_hx", info
    assert info["variant"] == variant
    np.testing.assert_array_equal(got["last_row"], ref.last_row)
    assert got["score"] == ref.score
    if tab:
        np.testing.assert_array_equal(got["table"], ref.table)


@pytest.mark.parametrize("variant", VARIANTS)
@pytest.mark.parametrize("shape", [(1000, 1000), (300, 2052), (33, 452)])
def test_min2plus_diagmaxplus_hx(hx_env, variant, shape):
    hx_env(variant)
    H, W = shape
    init = inputs.gen_init(H + 5 * W, H, W, hi=10000)
    ref = oracle.min2plus(init, 3, table=True)
    got = run_gpu("min2plus", "prev_row", grid=init, param_c=3, outputs=("score", "last_row", "table"))
    assert json.loads(got["plan"])["kernel"] == "prevrow_hx"
    np.testing.assert_array_equal(got["last_row"], ref.last_row)
    np.testing.assert_array_equal(got["table"], ref.table)
    assert got["score"] == ref.score
    ref = oracle.diagmaxplus(init, 2, table=True)
    got = run_gpu("diagmaxplus", "prev_row", grid=init, param_c=2, outputs=("last_row", "table"))
    assert json.loads(got["plan"])["kernel"] == "prevrow_hx"
    np.testing.assert_array_equal(got["last_row"], ref.last_row)
    np.testing.assert_array_equal(got["table"], ref.table)


@pytest.mark.parametrize("variant", [0, 2])
def test_hx_pitched_grid(hx_env, variant):
    """Row pitch > cols (a view into a wider grid): copies use the pitch, not the width."""
    hx_env(variant)
    c = inputs.gen_costs(5, 700, 1032)
    ref = oracle.minpath3(c)
    got = run_gpu("minpath3", "prev_row", grid=c, outputs=("score", "last_row"), grid_pad=12)
    assert json.loads(got["plan"])["kernel"] == "prevrow_hx"
    np.testing.assert_array_equal(got["last_row"], ref.last_row)
    assert got["score"] == ref.score


def test_hx_dispatch_rules(hx_env):
    """TABLE outputs run prevrow_hx too (16-byte row stores; a table pitch that is not a multiple
    of 4 falls back to prevrow_cb at fill time); an explicit band_rows keeps prevrow_cb;
    HX_VARIANT=-1 too."""
    hx_env(0)
    c = inputs.gen_costs(9, 300, 400)
    ref = oracle.minpath3(c, table=True)
    got = run_gpu("minpath3", "prev_row", grid=c, outputs=("score", "last_row", "table"))
    assert json.loads(got["plan"])["kernel"] == "prevrow_hx"
    np.testing.assert_array_equal(got["table"], ref.table)
    got = run_gpu("minpath3", "prev_row", grid=c, outputs=("score", "last_row", "table"), table_pad=3)
    np.testing.assert_array_equal(got["table"], ref.table)   # pitch 403: the prevrow_cb fill
    got = run_gpu("minpath3", "prev_row", grid=c, outputs=("score", "last_row"), band_rows=32)
    assert json.loads(got["plan"])["kernel"] == "prevrow_cb"
    assert got["score"] == ref.score
    hx_env(-1)
    got = run_gpu("minpath3", "prev_row", grid=c, outputs=("score", "last_row"))
    assert json.loads(got["plan"])["kernel"] == "prevrow_cb"
    np.testing.assert_array_equal(got["last_row"], ref.last_row)


def test_hx_full_width_c4_sample(hx_env):
    """C4's width (32768 columns: 147 CTAs of 224 on one B200, every CTA resident) over 600 rows."""
    hx_env(2)
    c = inputs.gen_costs(4, 600, 32768)
    ref = oracle.minpath3(c)
    got = run_gpu("minpath3", "prev_row", grid=c, outputs=("score", "last_row"))
    info = json.loads(got["plan"])
    assert info["kernel"] == "prevrow_hx" and info["grid"] == 147
    np.testing.assert_array_equal(got["last_row"], ref.last_row)
    assert got["score"] == ref.score


def test_hx_too_wide_falls_back(hx_env):
    """More CTAs than can be co-resident (W > 148 x 224 columns): the plan keeps prevrow_cb."""
    hx_env(2)
    c = inputs.gen_costs(6, 40, 40000)
    ref = oracle.minpath3(c)
    got = run_gpu("minpath3", "prev_row", grid=c, outputs=("score", "last_row"))
    assert json.loads(got["plan"])["kernel"] != "prevrow_hx"
    np.testing.assert_array_equal(got["last_row"], ref.last_row)
    assert got["score"] == ref.score
