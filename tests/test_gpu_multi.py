"""Multi-GPU column-strip fill (lddp_fill_multi) exercised on ONE GPU: P virtual ranks, each with
its own comm window, workspace and stream, chained with lddp_comm_connect_local.  The kernel
path is the same as across GPUs (peer stores of the strip's right column into rank g+1's window
+ system-scope release flags); only the pointer is local.  Results must equal the oracle."""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_kumark15_b200 import inputs

pytestmark = pytest.mark.gpu


def run_loopback(func, a, b, P, grid_per_rank=24, reps=2):
    import torch

    from paper_conf_ipps_kumark15_b200 import lddp

    dev = torch.device("cuda:0")
    m, n = len(a), len(b)
    cell = torch.float32 if func == "dtw" else torch.int32
    plan = lddp.Plan(func, "anti_diagonal", m, n,
                     lddp.OUT_SCORE | lddp.OUT_LAST_ROW | lddp.OUT_LAST_COL, grid_ctas=grid_per_rank)
    comms = [lddp.lddp_comm_create(plan.handle, P, g) for g in range(P)]
    for g in range(P):
        lddp.lddp_comm_connect_local(comms[g], comms[g + 1] if g + 1 < P else None)
    ta = torch.from_numpy(np.ascontiguousarray(a)).to(dev)
    tb = torch.from_numpy(np.ascontiguousarray(b)).to(dev)
    score = torch.full((1,), -7, dtype=cell, device=dev)
    last_row = torch.full((n,), -7, dtype=cell, device=dev)
    last_col = torch.full((m,), -7, dtype=cell, device=dev)
    wss = [torch.zeros(plan.ws_bytes, dtype=torch.uint8, device=dev) for _ in range(P)]
    streams = [torch.cuda.Stream(dev) for _ in range(P)]
    torch.cuda.synchronize()
    try:
        for _ in range(reps):
            for g in range(P):
                inp, out = plan.io(a=ta, b=tb, score=score, last_row=last_row, last_col=last_col)
                lddp.lddp_fill_multi(plan.handle, inp, out, wss[g].data_ptr(), comms[g],
                                     streams[g].cuda_stream)
            for g in range(P):
                lddp.lddp_status_check(plan.handle, wss[g].data_ptr(), streams[g].cuda_stream)
        torch.cuda.synchronize()
        return score.cpu().numpy()[0], last_row.cpu().numpy(), last_col.cpu().numpy()
    finally:
        for c in comms:
            lddp.lddp_comm_destroy(c)


@pytest.mark.parametrize("func", ["lcs", "levenshtein", "dtw"])
@pytest.mark.parametrize("P", [2, 3, 4])
@pytest.mark.parametrize("shape", [(700, 900), (1537, 1000), (2100, 4001)])
def test_loopback_column_strips(func, P, shape):
    m, n = shape
    if func == "dtw":
        a, b = inputs.gen_walks(m + n + P, m, n)
    else:
        a, b = inputs.gen_strings(m + n + P, m, n)
    ref = {"lcs": oracle.lcs, "levenshtein": oracle.levenshtein, "dtw": oracle.dtw}[func](a, b)
    s, lr, lc = run_loopback(func, a, b, P)
    if func == "dtw":
        assert s.tobytes() == np.float32(ref.score).tobytes()
        np.testing.assert_array_equal(lr.view(np.int32), ref.last_row.view(np.int32))
        np.testing.assert_array_equal(lc.view(np.int32), ref.last_col.view(np.int32))
    else:
        assert s == ref.score
        np.testing.assert_array_equal(lr, ref.last_row)
        np.testing.assert_array_equal(lc, ref.last_col)
