"""GPU traceback (csrc/traceback.cu) against the oracle's traceback of the
oracle's own table: the same DP cells, element by element (the GPU table is bit-exact, so the
tie-breaks see the same values), for LCS, Levenshtein and DTW at ragged shapes."""
import numpy as np
import pytest
import torch

import oracle
from paper_conf_ipps_kumark15_b200 import inputs, lddp

pytestmark = pytest.mark.gpu

SHAPES = [(1, 1), (1, 9), (9, 1), (7, 13), (64, 65), (300, 257), (1000, 700)]


@pytest.mark.parametrize("func", ["lcs", "levenshtein", "dtw"])
@pytest.mark.parametrize("shape", SHAPES)
def test_traceback_matches_oracle(func, shape):
    m, n = shape
    dev = torch.device("cuda:0")
    if func == "dtw":
        a, b = inputs.gen_walks(7 * m + n, m, n)
        ref = oracle.dtw(a, b, table=True)
        dt = torch.float32
    else:
        a, b = inputs.gen_strings(7 * m + n, m, n)
        ref = (oracle.lcs if func == "lcs" else oracle.levenshtein)(a, b, table=True)
        dt = torch.int32
    plan = lddp.Plan(func, "anti_diagonal", m, n, lddp.OUT_TABLE)
    ta, tb = torch.from_numpy(np.ascontiguousarray(a)).to(dev), torch.from_numpy(np.ascontiguousarray(b)).to(dev)
    table = torch.zeros((m, n + 3), dtype=dt, device=dev)[:, :n]
    plan.fill(a=ta, b=tb, table=table)
    plan.check()
    pi, pj = plan.traceback(ta, tb, table)
    got = list(zip(pi.cpu().tolist(), pj.cpu().tolist()))
    want = oracle.traceback(func, a, b, ref.table)
    assert got == want
    if func == "lcs":
        assert len(oracle.lcs_string(a, b, got)) == ref.score


def test_traceback_rejects_other_f():
    plan = lddp.Plan("minpath3", "prev_row", 8, 8, lddp.OUT_TABLE)
    t = torch.zeros((8, 8), dtype=torch.int32, device="cuda:0")
    with pytest.raises(lddp.LddpError):
        plan.traceback(t, t, t)
