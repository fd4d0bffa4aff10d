"""Batched Floyd-Steinberg (image-parallel, reading R21): B independent images
stacked along the rows, filled by ONE fsk launch whose warps claim (strip, image) pairs, and the
multi-GPU image shares of lddp_fill_multi (loopback ranks on one GPU).  Every image is compared
with the oracle's FS of that image alone ([L335-L348])."""
import ctypes
import json

import numpy as np
import pytest

import oracle
from paper_conf_ipps_kumark15_b200 import inputs

pytestmark = pytest.mark.gpu


def _batch(B, H, W, seed):
    imgs = [inputs.gen_image(seed + 7 * b, H, W, "ramp" if b % 2 else "uniform") for b in range(B)]
    return imgs, np.concatenate(imgs, axis=0)


@pytest.mark.parametrize("B", [1, 2, 3, 5, 9])
@pytest.mark.parametrize("shape", [(1, 16), (33, 64), (100, 160), (257, 512), (64, 1024)])
def test_fs_batch_one_launch(B, shape):
    import torch

    from paper_conf_ipps_kumark15_b200 import lddp
    H, W = shape
    imgs, stack = _batch(B, H, W, 3 * H + W)
    dev = torch.device("cuda:0")
    plan = lddp.Plan("fs", "knight_move", H, W, lddp.OUT_TABLE, batch=B)
    info = json.loads(plan.info)
    assert info["kernel"] == "fsk" and info["batch"] == B, info
    g = torch.from_numpy(stack).to(dev)
    out = torch.full_like(g, 77)
    for _ in range(2):   # two fills on one workspace (epoch-tagged boundary rows)
        plan.fill(grid=g, table=out)
    plan.check()
    got = out.cpu().numpy()
    for b in range(B):
        np.testing.assert_array_equal(got[b * H:(b + 1) * H], oracle.fs(imgs[b]), err_msg=f"image {b}")


def test_fs_batch_host_buffers():
    """lddp_fill_host copies the whole batch (B * H rows) both ways."""
    from paper_conf_ipps_kumark15_b200 import lddp
    B, H, W = 4, 70, 96
    imgs, stack = _batch(B, H, W, 11)
    plan = lddp.Plan("fs", "knight_move", H, W, lddp.OUT_TABLE, batch=B)
    out = np.zeros_like(stack)
    inp = lddp.lddp_inputs(grid=stack.ctypes.data_as(ctypes.c_void_p), grid_pitch=W)
    o = lddp.lddp_outputs(table=out.ctypes.data_as(ctypes.c_void_p), table_pitch=W)
    lddp.lddp_fill_host(plan.handle, inp, o)
    for b in range(B):
        np.testing.assert_array_equal(out[b * H:(b + 1) * H], oracle.fs(imgs[b]))


@pytest.mark.parametrize("P,B", [(2, 5), (3, 3), (4, 2), (3, 7)])
def test_fs_batch_multi_shares(P, B):
    """lddp_fill_multi: rank g fills images [g B / P, (g+1) B / P) (lddp_plan_partition), no
    exchange; the ranks' shares tile the batch."""
    import torch

    from paper_conf_ipps_kumark15_b200 import lddp
    H, W = 97, 128
    imgs, stack = _batch(B, H, W, 5 + P)
    dev = torch.device("cuda:0")
    plan = lddp.Plan("fs", "knight_move", H, W, lddp.OUT_TABLE, batch=B)
    comms = [lddp.lddp_comm_create(plan.handle, P, r) for r in range(P)]
    shares = [lddp.lddp_plan_partition(plan.handle, P, r) for r in range(P)]
    assert shares[0][0] == 0 and shares[-1][1] == B
    assert all(shares[r][1] == shares[r + 1][0] for r in range(P - 1))
    g = torch.from_numpy(stack).to(dev)
    out = torch.full_like(g, 77)
    wss = [torch.zeros(plan.ws_bytes, dtype=torch.uint8, device=dev) for _ in range(P)]
    streams = [torch.cuda.Stream(dev) for _ in range(P)]
    torch.cuda.synchronize()
    try:
        for r in range(P):
            inp, o = plan.io(grid=g, table=out)
            lddp.lddp_fill_multi(plan.handle, inp, o, wss[r].data_ptr(), comms[r], streams[r].cuda_stream)
        for r in range(P):
            lddp.lddp_status_check(plan.handle, wss[r].data_ptr(), streams[r].cuda_stream)
        torch.cuda.synchronize()
    finally:
        for c in comms:
            lddp.lddp_comm_destroy(c)
    got = out.cpu().numpy()
    for b in range(B):
        np.testing.assert_array_equal(got[b * H:(b + 1) * H], oracle.fs(imgs[b]), err_msg=f"image {b}")


def test_fs_batch_rejections():
    from paper_conf_ipps_kumark15_b200 import lddp
    with pytest.raises(lddp.LddpError):
        lddp.Plan("minpath3", "prev_row", 64, 64, lddp.OUT_SCORE, batch=2)
    with pytest.raises(lddp.LddpError):
        lddp.Plan("fs", "knight_move", 64, 100, lddp.OUT_TABLE, batch=2)   # cols % 16 != 0: no fsk
