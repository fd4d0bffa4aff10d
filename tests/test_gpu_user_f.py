"""GPU parity of user-supplied f's through the header-only lddp_user::fill<F>() (include/
lddp_user.cuh): the functors of tests/user_f/user_f.cu re-express paper f's with the user
interface, in every category whose schedule orders their declared contributing set (Table I),
and must equal the CPU oracle bit for bit ("a user needs to supply only the function f" [L45],
[L312])."""
import ctypes
import os

import numpy as np
import pytest

import oracle
from conftest import ROOT
from paper_conf_ipps_kumark15_b200 import inputs

pytestmark = pytest.mark.gpu
LIB = os.path.join(ROOT, "tests", "user_f", "libuserf.so")
PREV_ROW, ANTI_DIAGONAL, KNIGHT_MOVE, INVERTED_L = 0, 1, 2, 3


@pytest.fixture(scope="module")
def lib():
    ctypes.CDLL(os.path.join(ROOT, "paper_conf_ipps_kumark15_b200", "liblddp.so"), mode=ctypes.RTLD_GLOBAL)
    L = ctypes.CDLL(LIB)
    L.userf_ws_bytes.restype = ctypes.c_size_t
    L.userf_ws_bytes.argtypes = [ctypes.c_int, ctypes.c_int64, ctypes.c_int64, ctypes.c_int]
    L.userf_fill.restype = ctypes.c_int
    L.userf_fill.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64, ctypes.c_int] + \
        [ctypes.c_void_p] * 4 + [ctypes.c_int64, ctypes.c_void_p, ctypes.c_void_p]
    return L


def _fill(lib, which, user_words, keep, H, W, cat, want=("score", "last_row", "last_col", "table")):
    import torch
    dev = torch.device("cuda:0")
    user = torch.tensor(user_words, dtype=torch.int64, device=dev)
    out = {k: torch.full(shape, -7, dtype=torch.int32, device=dev) for k, shape in
           (("score", (1,)), ("last_row", (W,)), ("last_col", (H,)), ("table", (H, W + 3))) if k in want}
    ws = torch.zeros(lib.userf_ws_bytes(which, H, W, cat), dtype=torch.uint8, device=dev)
    p = lambda k: out[k].data_ptr() if k in out else None
    for _ in range(2):
        st = lib.userf_fill(which, user.data_ptr(), H, W, cat, p("score"), p("last_row"), p("last_col"), p("table"),
                            W + 3, ws.data_ptr(), torch.cuda.current_stream(dev).cuda_stream)
        assert st == 0, st
    torch.cuda.synchronize()
    del keep
    res = {k: v.cpu().numpy() for k, v in out.items()}
    if "table" in res:
        res["table"] = res["table"][:, :W]
    return res


SHAPES = [(1, 1), (7, 300), (300, 7), (513, 700), (1201, 333)]


@pytest.mark.parametrize("H,W", SHAPES)
@pytest.mark.parametrize("cat", [ANTI_DIAGONAL, KNIGHT_MOVE])
def test_user_lcs(lib, H, W, cat):
    import torch
    a, b = inputs.gen_strings(H * 3 + W, H, W)
    ta, tb = torch.from_numpy(a).cuda(), torch.from_numpy(b).cuda()
    ref = oracle.lcs(a, b, table=True)
    got = _fill(lib, 0, [ta.data_ptr(), tb.data_ptr()], (ta, tb), H, W, cat)
    assert got["score"][0] == ref.score
    np.testing.assert_array_equal(got["last_row"], ref.last_row)
    np.testing.assert_array_equal(got["last_col"], ref.last_col)
    np.testing.assert_array_equal(got["table"], ref.table)


@pytest.mark.parametrize("H,W", SHAPES)
@pytest.mark.parametrize("cat", [PREV_ROW, KNIGHT_MOVE])
def test_user_minpath(lib, H, W, cat):
    import torch
    c = inputs.gen_costs(H + W, H, W)
    tc = torch.from_numpy(c).cuda()
    ref = oracle.minpath3(c, table=True)
    want = ("score", "last_row", "table") if cat == PREV_ROW else ("score", "last_row", "last_col", "table")
    got = _fill(lib, 1, [tc.data_ptr(), W], tc, H, W, cat, want)
    assert got["score"][0] == ref.score
    np.testing.assert_array_equal(got["last_row"], ref.last_row)
    np.testing.assert_array_equal(got["table"], ref.table)


@pytest.mark.parametrize("H,W", SHAPES)
@pytest.mark.parametrize("which,cats,ref_fn", [
    (2, (ANTI_DIAGONAL, KNIGHT_MOVE), lambda g: oracle.min2plus_v(g, 1, table=True)),
    (3, (PREV_ROW, ANTI_DIAGONAL, KNIGHT_MOVE, INVERTED_L), lambda g: oracle.diagmaxplus(g, 1, table=True)),
    (4, (PREV_ROW, KNIGHT_MOVE), lambda g: oracle.antidiag_maxplus(g, 1, table=True)),
])
def test_user_synthetic_and_twins(lib, H, W, which, cats, ref_fn):
    """The Vertical / mInverted-L twins and the inverted-L f as user functors, in every category
    that orders their masks (schedule independence of the generic kernels)."""
    import torch
    g = inputs.gen_init(H * 11 + W + which, H, W)
    tg = torch.from_numpy(g).cuda()
    ref = ref_fn(g)
    for cat in cats:
        got = _fill(lib, which, [tg.data_ptr(), W, W], tg, H, W, cat, ("table",))
        np.testing.assert_array_equal(got["table"], ref.table, err_msg=f"category {cat}")
