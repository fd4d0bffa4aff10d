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


def test_traceback_at_100k_full_table_in_hbm():
    """SURVEY 8(f)#2 at the C5 size: the whole 100000 x 100000 int32 LCS table (40 GB) fits in one
    B200's HBM, so the traceback is a TABLE fill plus the device walk -- no linear-space
    (Hirschberg) recursion is needed on this part.  Checked against the
    oracle's full-size LCS length (tests/golden/bench_refs.json, C5) and by the path itself: it
    is monotone from (m, n) to the boundary, and its diagonal match steps spell a common
    subsequence of a and b of exactly that length."""
    import json
    import os

    free, _ = torch.cuda.mem_get_info()
    if free < 44 << 30:
        pytest.skip("needs ~44 GB of free device memory")
    n = 100000
    a, b = inputs.gen_strings(0, n, n)   # C5's inputs (tools/configs.py, seed 0)
    with open(os.path.join(os.path.dirname(__file__), "golden", "bench_refs.json")) as f:
        want = json.load(f)["configs"]["C5"]["score"]
    dev = torch.device("cuda:0")
    ta, tb = torch.from_numpy(a).to(dev), torch.from_numpy(b).to(dev)
    table = torch.empty((n, n), dtype=torch.int32, device=dev)
    plan = lddp.Plan("lcs", "anti_diagonal", n, n, lddp.OUT_TABLE)
    plan.fill(a=ta, b=tb, table=table)
    plan.check()
    assert int(table[n - 1, n - 1].item()) == want
    pi, pj = plan.traceback(ta, tb, table)
    del table
    i, j = pi.cpu().numpy().astype(np.int64), pj.cpu().numpy().astype(np.int64)
    assert i[0] == n and j[0] == n and (i.min() == 1 or j.min() == 1)
    di, dj = i[:-1] - i[1:], j[:-1] - j[1:]
    assert np.all(((di == 1) & (dj == 1)) | ((di == 1) & (dj == 0)) | ((di == 0) & (dj == 1)))
    # a diagonal step out of cell (i, j) is taken exactly on a match a_i == b_j (CLRS, R14); the
    # last cell of the path steps to the boundary, diagonally iff it matches
    diag = np.concatenate([(di == 1) & (dj == 1), [a[i[-1] - 1] == b[j[-1] - 1]]])
    mi, mj = i[diag] - 1, j[diag] - 1
    assert np.array_equal(a[mi], b[mj])
    assert int(diag.sum()) == want
