"""Host-side tests of the header-only user-f API (include/lddp_user.cuh): the example functors of
tests/user_f/user_f.cu compile against the library's kernel templates, and lddp_user::check()
applies Table I [L124-L142] + the Fig. 2 schedules to a user's declared contributing set (no GPU)."""
import ctypes
import os

import pytest

from conftest import ROOT

LIB = os.path.join(ROOT, "tests", "user_f", "libuserf.so")
PREV_ROW, ANTI_DIAGONAL, KNIGHT_MOVE, INVERTED_L = 0, 1, 2, 3
OK, CATEGORY_MISMATCH, UNSUPPORTED = 0, 3, 4
# (functor id, categories whose schedule orders its mask)
ORDERED = {0: {ANTI_DIAGONAL, KNIGHT_MOVE},                 # LCS {L, UL, U}
           1: {PREV_ROW, KNIGHT_MOVE},                      # min-path {UL, U, UR}
           2: {ANTI_DIAGONAL, KNIGHT_MOVE},                 # Vertical twin {L, UL}
           3: {PREV_ROW, ANTI_DIAGONAL, KNIGHT_MOVE, INVERTED_L},   # {UL}
           4: {PREV_ROW, KNIGHT_MOVE}}                      # mInverted-L twin {UR}


@pytest.fixture(scope="module")
def lib():
    if not os.path.exists(LIB):
        pytest.skip("tests/user_f/libuserf.so not built (make -C paper_conf_ipps_kumark15_b200)")
    ctypes.CDLL(os.path.join(ROOT, "paper_conf_ipps_kumark15_b200", "liblddp.so"), mode=ctypes.RTLD_GLOBAL)
    L = ctypes.CDLL(LIB)
    L.userf_check.restype = ctypes.c_int
    L.userf_check.argtypes = [ctypes.c_int, ctypes.c_int]
    L.userf_ws_bytes.restype = ctypes.c_size_t
    L.userf_ws_bytes.argtypes = [ctypes.c_int, ctypes.c_int64, ctypes.c_int64, ctypes.c_int]
    return L


def test_check_applies_table1(lib):
    for which, ok_cats in ORDERED.items():
        for cat in (PREV_ROW, ANTI_DIAGONAL, KNIGHT_MOVE, INVERTED_L):
            st = lib.userf_check(which, cat)
            assert st == (OK if cat in ok_cats else CATEGORY_MISMATCH), (which, cat, st)
        assert lib.userf_check(which, 4) == UNSUPPORTED   # twins: through knight-move


def test_workspace_sizes(lib):
    for which, cats in ORDERED.items():
        for cat in cats:
            assert lib.userf_ws_bytes(which, 1000, 777, cat) >= 64
