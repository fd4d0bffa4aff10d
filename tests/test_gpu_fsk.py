"""GPU parity of the lane-systolic Floyd-Steinberg kernel (csrc/fsk.cu) against the CPU oracle,
bit-exact (uint8 output image): widths that are multiples of 16 (the kernel's precondition; other
widths and 16-byte-unaligned pitches take the wavefront fallback, also checked), heights that
leave ragged last strips, every compiled (warps, extra lag), repeated fills on one workspace."""
import json
import os

import numpy as np
import pytest

import oracle
from gpu_util import run_gpu
from paper_conf_ipps_kumark15_b200 import inputs

pytestmark = pytest.mark.gpu

FS_SHAPES = [(1, 16), (2, 32), (3, 16), (7, 48), (33, 64), (100, 160), (129, 256), (257, 512),
             (300, 1024), (64, 4096), (1000, 2048)]


@pytest.fixture
def fsk_env():
    keys = ("LDDP_FSK", "LDDP_FSK_W", "LDDP_FSK_E", "LDDP_FSK_R")
    old = {k: os.environ.get(k) for k in keys}

    def set_(w, e, on=1, r=1):
        os.environ["LDDP_FSK"], os.environ["LDDP_FSK_W"], os.environ["LDDP_FSK_E"] = str(on), str(w), str(e)
        os.environ["LDDP_FSK_R"] = str(r)

    yield set_
    for k, v in old.items():
        if v is None:
            os.environ.pop(k, None)
        else:
            os.environ[k] = v


@pytest.mark.parametrize("w,e,r", [(1, 1, 1), (1, 0, 1), (1, 2, 1), (1, 1, 2), (1, 0, 2), (4, 1, 1), (2, 1, 1)])
@pytest.mark.parametrize("shape", FS_SHAPES)
@pytest.mark.parametrize("kind", ["ramp", "uniform"])
def test_fsk_parity(fsk_env, w, e, r, shape, kind):
    fsk_env(w, e, r=r)
    H, W = shape
    img = inputs.gen_image(11 * H + W, H, W, kind)
    ref = oracle.fs(img)
    got = run_gpu("fs", "knight_move", grid=img, outputs=("table",), reps=2)
    info = json.loads(got["plan"])
    assert info["kernel"] == "fsk", info
    np.testing.assert_array_equal(got["table"], ref)


def test_fsk_fallback_width(fsk_env):
    """W % 16 != 0: the wavefront kernel, same bits."""
    fsk_env(4, 1)
    img = inputs.gen_image(5, 100, 200 + 4, "ramp")
    got = run_gpu("fs", "knight_move", grid=img, outputs=("table",))
    assert json.loads(got["plan"])["kernel"] == "wavefront"
    np.testing.assert_array_equal(got["table"], oracle.fs(img))


def test_fsk_fallback_pitch(fsk_env):
    """W % 16 == 0 but a table pitch that is not a 16-byte multiple: wavefront fallback per fill."""
    fsk_env(4, 1)
    img = inputs.gen_image(6, 90, 160, "uniform")
    got = run_gpu("fs", "knight_move", grid=img, outputs=("table",), table_pad=4)
    np.testing.assert_array_equal(got["table"], oracle.fs(img))
