"""Device watchdog: a dependency that never arrives must end the kernel with LDDP_ERR_TIMEOUT
(reported by lddp_status_check) instead of hanging the GPU.  Rank 1 of a 2-rank column-strip
fill is launched alone, so it waits forever for rank 0's boundary column."""
import os

import numpy as np
import pytest

from paper_conf_ipps_kumark15_b200 import inputs

pytestmark = pytest.mark.gpu


def test_missing_left_neighbour_times_out():
    import torch

    from paper_conf_ipps_kumark15_b200 import lddp

    os.environ["LDDP_TIMEOUT_MS"] = "300"
    try:
        dev = torch.device("cuda:0")
        a, b = inputs.gen_strings(0, 1000, 600)
        plan = lddp.Plan("lcs", "anti_diagonal", 1000, 600, lddp.OUT_SCORE | lddp.OUT_LAST_ROW, grid_ctas=8)
        c0 = lddp.lddp_comm_create(plan.handle, 2, 0)
        c1 = lddp.lddp_comm_create(plan.handle, 2, 1)
        lddp.lddp_comm_connect_local(c0, c1, None)
        lddp.lddp_comm_connect_local(c1, None, c0)
        ta, tb = torch.from_numpy(a).to(dev), torch.from_numpy(b).to(dev)
        score = torch.zeros(1, dtype=torch.int32, device=dev)
        lr = torch.zeros(600, dtype=torch.int32, device=dev)
        inp, out = plan.io(a=ta, b=tb, score=score, last_row=lr)
        s = torch.cuda.current_stream(dev)
        lddp.lddp_fill_multi(plan.handle, inp, out, plan.ws.data_ptr(), c1, s.cuda_stream)   # rank 1 only
        with pytest.raises(lddp.LddpError) as e:
            lddp.lddp_status_check(plan.handle, plan.ws.data_ptr(), s.cuda_stream)
        assert e.value.status == lddp.LDDP_ERR_TIMEOUT
        # the workspace is usable again: a normal single-GPU fill on it succeeds
        os.environ["LDDP_TIMEOUT_MS"] = "30000"
        plan.fill(a=ta, b=tb, score=score, last_row=lr)
        plan.check()
        import oracle
        assert int(score.item()) == oracle.lcs(a, b).score
        lddp.lddp_comm_destroy(c0)
        lddp.lddp_comm_destroy(c1)
    finally:
        os.environ.pop("LDDP_TIMEOUT_MS", None)
