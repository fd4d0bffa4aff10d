"""Host-side tests of the C ABI (no GPU needed): the library loads, exports every symbol that
include/lddp.h declares, and its classifier / category-coverage logic matches Table I and the
Fig. 2 schedules."""
import ctypes
import os
import re
import subprocess

import pytest

from conftest import ROOT, golden
from test_oracle_pins import OFFSETS, schedule_valid

HEADER = os.path.join(ROOT, "include", "lddp.h")
LIB = os.path.join(ROOT, "paper_conf_ipps_kumark15_b200", "liblddp.so")


@pytest.fixture(scope="module")
def lddp():
    if not os.path.exists(LIB):
        subprocess.check_call(["make", "-C", os.path.dirname(LIB), "-j8"])
    from paper_conf_ipps_kumark15_b200 import lddp as mod
    return mod


def header_functions():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(lddp_[a-z_]+)\s*\(", text)))


def test_header_symbols_exported(lddp):
    names = header_functions()
    assert len(names) >= 20
    lib = ctypes.CDLL(LIB)
    for name in names:
        assert hasattr(lib, name), f"{name} declared in include/lddp.h but not exported"
    # the binding wraps exactly the header's functions
    assert sorted(lddp.EXPORTED) == names


def test_abi_version_and_strings(lddp):
    assert lddp.lddp_abi_version() == 2
    for st, name in lddp.STATUS_NAMES.items():
        assert lddp._lib.lddp_status_string(st).decode() == name


def test_classify_matches_table1(lddp):
    names = {v: k for k, v in lddp.PATTERN_NAMES.items()}
    for row in golden("table1.json")["rows"]:
        mask = sum(bit for key, bit in (("L", 1), ("UL", 2), ("U", 4), ("UR", 8)) if row[key] == "Y")
        assert lddp.lddp_classify(mask) == names[row["pattern"]], row


CAT_PATTERN = {0: "Horizontal", 1: "Anti-diagonal", 2: "Knight-Move", 3: "Inverted-L", 4: "Vertical",
               5: "mInverted-L"}


def test_category_covers_matches_schedules(lddp):
    """covers(category, mask) must equal 'the category's Fig. 2 schedule strictly orders every
    dependency of the mask' -- checked by brute force on a 7x7 grid."""
    for cat, pat in CAT_PATTERN.items():
        for mask in range(1, 16):
            nbs = [k for k, bit in (("L", 1), ("UL", 2), ("U", 4), ("UR", 8)) if mask & bit]
            assert lddp.lddp_category_covers(cat, mask) == schedule_valid(pat, nbs), (cat, mask)


def test_func_masks(lddp):
    assert lddp.lddp_func_mask(lddp.F_LCS) == 1 | 2 | 4          # Fig. 1(c) [L88]
    assert lddp.lddp_func_mask(lddp.F_LEVENSHTEIN) == 1 | 2 | 4  # [L327]
    assert lddp.lddp_func_mask(lddp.F_FS_DITHER) == 15           # [L341-L344]
    assert lddp.lddp_func_mask(lddp.F_MIN_PATH3) == 2 | 4 | 8    # [L365]
    assert lddp.lddp_func_mask(lddp.F_DIAG_MAXPLUS) == 2         # [L298]
    assert lddp.lddp_func_mask(lddp.F_MIN2_PLUS) == 2 | 4        # [L298]
    assert lddp.lddp_func_mask(lddp.F_MIN2_PLUS_V) == 1 | 2      # Vertical twin [L111], R15
    assert lddp.lddp_func_mask(lddp.F_ANTIDIAG_MAXPLUS) == 8     # mInverted-L twin [L111], R15
    # Table I classifies each compiled f into the pattern of the category it runs in
    assert lddp.lddp_classify(lddp.lddp_func_mask(lddp.F_MIN2_PLUS_V)) == lddp.PAT_VERTICAL
    assert lddp.lddp_classify(lddp.lddp_func_mask(lddp.F_ANTIDIAG_MAXPLUS)) == lddp.PAT_MINVERTED_L
    with pytest.raises(lddp.LddpError):
        lddp.lddp_func_mask(99)


def test_plan_rejects_category_mismatch_without_gpu(lddp):
    """Argument validation happens before any device query."""
    d = lddp.lddp_desc(rows=10, cols=10, category=lddp.CAT_PREV_ROW, func=lddp.F_LCS,
                       outputs=lddp.OUT_SCORE)
    with pytest.raises(lddp.LddpError) as e:
        lddp.lddp_plan(d)
    assert e.value.status == lddp.LDDP_ERR_CATEGORY_MISMATCH
    d = lddp.lddp_desc(rows=10, cols=10, category=lddp.CAT_ANTI_DIAGONAL, func=lddp.F_FS_DITHER,
                       outputs=lddp.OUT_TABLE)
    with pytest.raises(lddp.LddpError) as e:
        lddp.lddp_plan(d)
    assert e.value.status == lddp.LDDP_ERR_CATEGORY_MISMATCH
    for cat, func in ((lddp.CAT_INVERTED_L, lddp.F_ANTIDIAG_MAXPLUS), (lddp.CAT_PREV_ROW, lddp.F_MIN2_PLUS_V)):
        d = lddp.lddp_desc(rows=10, cols=10, category=cat, func=func, outputs=lddp.OUT_LAST_ROW)
        with pytest.raises(lddp.LddpError) as e:   # {UR} / {L,UL} not ordered by these schedules
            lddp.lddp_plan(d)
        assert e.value.status == lddp.LDDP_ERR_CATEGORY_MISMATCH
    d = lddp.lddp_desc(rows=10, cols=10, category=lddp.CAT_ANTI_DIAGONAL, func=lddp.F_MIN2_PLUS_V,
                       outputs=lddp.OUT_SCORE)
    with pytest.raises(lddp.LddpError) as e:       # ordered, but the twin f runs on its twin's kernel
        lddp.lddp_plan(d)
    assert e.value.status == lddp.LDDP_ERR_UNSUPPORTED
    d = lddp.lddp_desc(rows=-1, cols=10, category=lddp.CAT_ANTI_DIAGONAL, func=lddp.F_LCS,
                       outputs=lddp.OUT_SCORE)
    with pytest.raises(lddp.LddpError) as e:
        lddp.lddp_plan(d)
    assert e.value.status == lddp.LDDP_ERR_SHAPE
