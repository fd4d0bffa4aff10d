"""Multi-GPU column-strip fill (lddp_fill_multi) exercised on ONE GPU.

* Loopback: P virtual ranks in one process, each with its own comm window, workspace and stream,
  chained with lddp_comm_connect_local.  The kernel path is the one used across GPUs (peer stores
  of each strip's right column into rank g+1's window slot, system-scope flags, consumer acks).
* Every fill of a test uses DIFFERENT inputs and outputs, and the fills are enqueued rank by rank
  (all fills of rank 0 before any fill of rank 1, ...), so producers run up to two fills ahead of
  their consumers: a receive window reused without back-pressure would hand rank g+1 the wrong
  fill's column.  Each result must equal the oracle.
* Cross-process: 2-3 processes on the same GPU exchange CUDA IPC window handles over a gloo
  process group (lddp_comm_handle / lddp_comm_connect), the path bench.py takes across GPUs."""
import json
import os
import socket
import time

import numpy as np
import pytest

import oracle
from paper_conf_ipps_kumark15_b200 import inputs

pytestmark = pytest.mark.gpu

REF = {"lcs": oracle.lcs, "levenshtein": oracle.levenshtein, "dtw": oracle.dtw}


def _inputs(func, seed, m, n):
    return inputs.gen_walks(seed, m, n) if func == "dtw" else inputs.gen_strings(seed, m, n)


def _check(func, got, ref):
    s, lr, lc = got
    if func == "dtw":
        assert np.float32(s).tobytes() == np.float32(ref.score).tobytes()
        np.testing.assert_array_equal(lr.view(np.int32), ref.last_row.view(np.int32))
        np.testing.assert_array_equal(lc.view(np.int32), ref.last_col.view(np.int32))
    else:
        assert s == ref.score
        np.testing.assert_array_equal(lr, ref.last_row)
        np.testing.assert_array_equal(lc, ref.last_col)


def run_loopback(func, problems, P, grid_per_rank=16, delay_ranks=0.0, kernel=None):
    """problems: list of (a, b), one fill each.  Returns [(score, last_row, last_col)]."""
    import torch

    from paper_conf_ipps_kumark15_b200 import lddp

    old = os.environ.get("LDDP_KERNEL")
    if kernel:
        os.environ["LDDP_KERNEL"] = kernel
    dev = torch.device("cuda:0")
    m, n = len(problems[0][0]), len(problems[0][1])
    cell = torch.float32 if func == "dtw" else torch.int32
    try:
        plan = lddp.Plan(func, "anti_diagonal", m, n,
                         lddp.OUT_SCORE | lddp.OUT_LAST_ROW | lddp.OUT_LAST_COL, grid_ctas=grid_per_rank)
    finally:
        if kernel:
            if old is None:
                os.environ.pop("LDDP_KERNEL", None)
            else:
                os.environ["LDDP_KERNEL"] = old
    comms = [lddp.lddp_comm_create(plan.handle, P, g) for g in range(P)]
    for g in range(P):
        lddp.lddp_comm_connect_local(comms[g], comms[g + 1] if g + 1 < P else None, comms[g - 1] if g > 0 else None)
    tens = [(torch.from_numpy(np.ascontiguousarray(a)).to(dev), torch.from_numpy(np.ascontiguousarray(b)).to(dev))
            for a, b in problems]
    outs = [(torch.full((1,), -7, dtype=cell, device=dev), torch.full((n,), -7, dtype=cell, device=dev),
             torch.full((m,), -7, dtype=cell, device=dev)) for _ in problems]
    wss = [torch.zeros(plan.ws_bytes, dtype=torch.uint8, device=dev) for _ in range(P)]
    streams = [torch.cuda.Stream(dev) for _ in range(P)]
    torch.cuda.synchronize()
    try:
        for g in range(P):   # rank by rank: rank g enqueues every fill before rank g+1 starts
            for (ta, tb), (sc, lr, lc) in zip(tens, outs):
                inp, out = plan.io(a=ta, b=tb, score=sc, last_row=lr, last_col=lc)
                lddp.lddp_fill_multi(plan.handle, inp, out, wss[g].data_ptr(), comms[g], streams[g].cuda_stream)
            if delay_ranks:
                time.sleep(delay_ranks)
        for g in range(P):
            lddp.lddp_status_check(plan.handle, wss[g].data_ptr(), streams[g].cuda_stream)
        torch.cuda.synchronize()
        return [(sc.cpu().numpy()[0], lr.cpu().numpy(), lc.cpu().numpy()) for sc, lr, lc in outs]
    finally:
        for c in comms:
            lddp.lddp_comm_destroy(c)


@pytest.mark.parametrize("func", ["lcs", "levenshtein", "dtw"])
@pytest.mark.parametrize("P", [2, 3, 4])
@pytest.mark.parametrize("shape", [(700, 900), (1537, 1000), (2100, 4001)])
def test_loopback_column_strips(func, P, shape):
    """Four fills with different inputs, enqueued rank by rank (producers run ahead)."""
    m, n = shape
    probs = [_inputs(func, 100 * k + m + n + P, m, n) for k in range(4)]
    for got, (a, b) in zip(run_loopback(func, probs, P), probs):
        _check(func, got, REF[func](a, b))


@pytest.mark.parametrize("kernel", ["adiag", None])
def test_loopback_back_pressure(kernel):
    """Rank 1 starts only after rank 0 has enqueued (and started) five fills: rank 0's third fill
    must wait on the GPU for rank 1's acknowledgement of the first before reusing its window slot."""
    probs = [_inputs("lcs", 7 * k + 1, 1000, 800) for k in range(5)]
    for got, (a, b) in zip(run_loopback("lcs", probs, 2, delay_ranks=0.2, kernel=kernel), probs):
        _check("lcs", got, oracle.lcs(a, b))


@pytest.mark.parametrize("P", [2, 3])
def test_loopback_adiag_dtw_lev(P):
    """The 32-bit adiag kernel's window path (LCS forced onto it too)."""
    for func, kernel in (("lcs", "adiag"), ("levenshtein", None), ("dtw", None)):
        probs = [_inputs(func, 31 * k + P, 1200, 700) for k in range(3)]
        for got, (a, b) in zip(run_loopback(func, probs, P, kernel=kernel), probs):
            _check(func, got, REF[func](a, b))


# ------------------------------------------------------------------------------ cross-process
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _ipc_rank(rank, world, port, func, m, n, fills, q):
    import torch
    import torch.distributed as dist

    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_kumark15_b200 import inputs as inp_mod
    from paper_conf_ipps_kumark15_b200 import lddp
    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    cell = torch.float32 if func == "dtw" else torch.int32
    plan = lddp.Plan(func, "anti_diagonal", m, n, lddp.OUT_SCORE | lddp.OUT_LAST_ROW | lddp.OUT_LAST_COL,
                     grid_ctas=8)
    comm = lddp.lddp_comm_create(plan.handle, world, rank)
    handles = [None] * world
    dist.all_gather_object(handles, lddp.lddp_comm_handle(comm))
    lddp.lddp_comm_connect(comm, handles[rank + 1] if rank + 1 < world else None,
                           handles[rank - 1] if rank > 0 else None)
    dist.barrier()
    c0, c1 = lddp.lddp_multi_partition(n, world, rank)
    res = []
    bufs = []
    stream = torch.cuda.current_stream(dev)
    if rank == 1:
        time.sleep(0.5)   # rank 0 runs ahead: its later fills must wait for rank 1's acks
    for k in range(fills):
        a, b = (inp_mod.gen_walks if func == "dtw" else inp_mod.gen_strings)(1000 + 17 * k, m, n)
        ta, tb = torch.from_numpy(a).to(dev), torch.from_numpy(b).to(dev)
        sc = torch.full((1,), -7, dtype=cell, device=dev)
        lr = torch.full((n,), -7, dtype=cell, device=dev)
        lc = torch.full((m,), -7, dtype=cell, device=dev)
        inp, out = plan.io(a=ta, b=tb, score=sc, last_row=lr, last_col=lc)
        lddp.lddp_fill_multi(plan.handle, inp, out, plan.ws.data_ptr(), comm, stream.cuda_stream)
        bufs.append((ta, tb, sc, lr, lc))
    lddp.lddp_status_check(plan.handle, plan.ws.data_ptr(), stream.cuda_stream)
    for ta, tb, sc, lr, lc in bufs:
        res.append((float(sc.cpu().numpy()[0]), lr.cpu().numpy()[c0:c1].tolist(),
                    lc.cpu().numpy().tolist() if rank == world - 1 else None))
    dist.barrier()
    lddp.lddp_comm_destroy(comm)
    q.put((rank, c0, c1, res))
    dist.destroy_process_group()


@pytest.mark.parametrize("func,world", [("lcs", 2), ("lcs", 3), ("dtw", 2)])
def test_cross_process_ipc(func, world):
    import torch.multiprocessing as mp
    m, n, fills = 900, 700, 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_ipc_rank, args=(r, world, port, func, m, n, fills, q)) for r in range(world)]
    for p in procs:
        p.start()
    parts = sorted([q.get(timeout=300) for _ in range(world)])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for k in range(fills):
        a, b = (inputs.gen_walks if func == "dtw" else inputs.gen_strings)(1000 + 17 * k, m, n)
        ref = REF[func](a, b)
        last = np.zeros(n, ref.last_row.dtype)
        for rank, c0, c1, res in parts:
            last[c0:c1] = np.asarray(res[k][1], ref.last_row.dtype)
        score = parts[-1][3][k][0]
        lcol = np.asarray(parts[-1][3][k][2], ref.last_col.dtype)
        _check(func, (np.asarray(score, ref.last_row.dtype), last, lcol), ref)


# ------------------------------------------------------------------ inverted-L diagonal shares
@pytest.mark.parametrize("func,cat", [("diagmaxplus", "inverted_l"), ("antidiag_maxplus", "minverted_l")])
@pytest.mark.parametrize("P", [1, 2, 3, 8])
@pytest.mark.parametrize("shape", [(1, 1), (700, 900), (1537, 100), (64, 3000)])
def test_inverted_l_diagonal_shares(func, cat, P, shape):
    """Inverted-L chains are independent ([L203]): each rank fills a contiguous share of the
    diagonals (equal cells), no window traffic; the union of the ranks' outputs equals the oracle."""
    import torch

    from paper_conf_ipps_kumark15_b200 import lddp
    H, W = shape
    g = inputs.gen_init(H + 3 * W + P, H, W)
    ref = (oracle.diagmaxplus if func == "diagmaxplus" else oracle.antidiag_maxplus)(g, 1, table=True)
    dev = torch.device("cuda:0")
    plan = lddp.Plan(func, cat, H, W, lddp.OUT_LAST_ROW | lddp.OUT_LAST_COL | lddp.OUT_TABLE)
    comms = [lddp.lddp_comm_create(plan.handle, P, r) for r in range(P)]
    tg = torch.from_numpy(g).to(dev)
    lr = torch.full((W,), -7, dtype=torch.int32, device=dev)
    lc = torch.full((H,), -7, dtype=torch.int32, device=dev)
    tab = torch.full((H, W), -7, dtype=torch.int32, device=dev)
    wss = [torch.zeros(max(plan.ws_bytes, 64), dtype=torch.uint8, device=dev) for _ in range(P)]
    try:
        for r in range(P):   # no connect needed: no exchange
            inp, out = plan.io(grid=tg, last_row=lr, last_col=lc, table=tab)
            lddp.lddp_fill_multi(plan.handle, inp, out, wss[r].data_ptr(), comms[r], 0)
        torch.cuda.synchronize()
        np.testing.assert_array_equal(tab.cpu().numpy(), ref.table)
        np.testing.assert_array_equal(lr.cpu().numpy(), ref.last_row)
        np.testing.assert_array_equal(lc.cpu().numpy(), ref.last_col)
    finally:
        for c in comms:
            lddp.lddp_comm_destroy(c)


# --------------------------------------------------- prev-row column strips, two-way halos
@pytest.mark.parametrize("func", ["minpath3", "min2plus"])
@pytest.mark.parametrize("P", [2, 3, 4])
@pytest.mark.parametrize("shape", [(300, 1024), (1000, 2048), (517, 1540), (64, 4096)])
@pytest.mark.parametrize("kernel", ["prevrow_hx", "prevrow_cb"])
def test_prev_row_two_way_halos(func, P, shape, kernel, monkeypatch):
    """Previous-row category across P ranks (loopback: all ranks on this GPU, each with its own
    window, workspace and stream), on both prev-row kernels: CTA- / block-aligned column strips; every band the strips' outer
    blocks exchange their HB-column edges with the neighbour ranks both ways (Table II case 2,
    [L193-L195], [L265-L274]).  Several fills with different grids, enqueued rank by rank.  The
    score is per rank (the minimum of its columns); its minimum over ranks is the oracle's."""
    import torch

    from paper_conf_ipps_kumark15_b200 import lddp
    H, W = shape
    dev = torch.device("cuda:0")
    if kernel == "prevrow_cb":   # the hierarchical-exchange kernel is the default when it fits
        monkeypatch.setenv("LDDP_HX_VARIANT", "-1")
    plan = lddp.Plan(func, "prev_row", H, W, lddp.OUT_SCORE | lddp.OUT_LAST_ROW | lddp.OUT_TABLE)
    assert json.loads(plan.info)["kernel"] == kernel
    comms = [lddp.lddp_comm_create(plan.handle, P, r) for r in range(P)]
    for r in range(P):
        lddp.lddp_comm_connect_local(comms[r], comms[r + 1] if r + 1 < P else None, comms[r - 1] if r > 0 else None)
    grids = [(inputs.gen_costs if func == "minpath3" else inputs.gen_init)(17 * k + P + H, H, W) for k in range(3)]
    tg = [torch.from_numpy(g).to(dev) for g in grids]
    outs = [(torch.full((P,), -7, dtype=torch.int32, device=dev), torch.full((W,), -7, dtype=torch.int32, device=dev),
             torch.full((H, W), -7, dtype=torch.int32, device=dev)) for _ in grids]
    wss = [torch.zeros(plan.ws_bytes, dtype=torch.uint8, device=dev) for _ in range(P)]
    streams = [torch.cuda.Stream(dev) for _ in range(P)]
    torch.cuda.synchronize()
    try:
        for r in range(P):
            for g, (sc, lr, tab) in zip(tg, outs):
                inp, out = plan.io(grid=g, score=sc[r:r + 1], last_row=lr, table=tab)
                lddp.lddp_fill_multi(plan.handle, inp, out, wss[r].data_ptr(), comms[r], streams[r].cuda_stream)
        for r in range(P):
            lddp.lddp_status_check(plan.handle, wss[r].data_ptr(), streams[r].cuda_stream)
        torch.cuda.synchronize()
        for g, (sc, lr, tab) in zip(grids, outs):
            ref = (oracle.minpath3(g, table=True) if func == "minpath3" else oracle.min2plus(g, 1, table=True))
            np.testing.assert_array_equal(tab.cpu().numpy(), ref.table)
            np.testing.assert_array_equal(lr.cpu().numpy(), ref.last_row)
            s = sc.cpu().numpy()
            for r in range(P):
                c0, c1 = lddp.lddp_plan_partition(plan.handle, P, r)
                assert c0 % 4 == 0 and (c1 == W or c1 % 4 == 0)
                if c1 > c0:
                    assert s[r] == ref.last_row[c0:c1].min()
            assert s[s != -7].min() == ref.score
    finally:
        for c in comms:
            lddp.lddp_comm_destroy(c)


def _ipc_rank_rows(rank, world, port, func, m, n, fills, q):
    """One process per rank (all on cuda:0): prev-row column strips through CUDA IPC windows."""
    import torch
    import torch.distributed as dist

    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_kumark15_b200 import inputs as inp_mod
    from paper_conf_ipps_kumark15_b200 import lddp
    dev = torch.device("cuda:0")
    torch.cuda.set_device(dev)
    plan = lddp.Plan(func, "prev_row", m, n, lddp.OUT_SCORE | lddp.OUT_LAST_ROW)
    comm = lddp.lddp_comm_create(plan.handle, world, rank)
    handles = [None] * world
    dist.all_gather_object(handles, lddp.lddp_comm_handle(comm))
    lddp.lddp_comm_connect(comm, handles[rank + 1] if rank + 1 < world else None,
                           handles[rank - 1] if rank > 0 else None)
    dist.barrier()
    c0, c1 = lddp.lddp_plan_partition(plan.handle, world, rank)
    stream = torch.cuda.current_stream(dev)
    if rank == 1:
        time.sleep(0.5)   # rank 0's kernel waits at its first band exchange
    bufs = []
    gen = inp_mod.gen_costs if func == "minpath3" else inp_mod.gen_init
    for k in range(fills):
        g = torch.from_numpy(gen(2000 + 17 * k, m, n)).to(dev)
        sc = torch.full((1,), -7, dtype=torch.int32, device=dev)
        lr = torch.full((n,), -7, dtype=torch.int32, device=dev)
        inp, out = plan.io(grid=g, score=sc, last_row=lr)
        lddp.lddp_fill_multi(plan.handle, inp, out, plan.ws.data_ptr(), comm, stream.cuda_stream)
        bufs.append((g, sc, lr))
    lddp.lddp_status_check(plan.handle, plan.ws.data_ptr(), stream.cuda_stream)
    res = [(int(sc.cpu().numpy()[0]), lr.cpu().numpy()[c0:c1].tolist()) for g, sc, lr in bufs]
    dist.barrier()
    lddp.lddp_comm_destroy(comm)
    q.put((rank, c0, c1, res))
    dist.destroy_process_group()


@pytest.mark.parametrize("func,world", [("minpath3", 2), ("minpath3", 3), ("min2plus", 2)])
def test_cross_process_ipc_prev_row(func, world):
    """Prev-row two-way halos between PROCESSES (CUDA IPC windows, handles over gloo), three
    back-to-back fills with different grids; strips from lddp_plan_partition tile [0, n)."""
    import torch.multiprocessing as mp
    m, n, fills = 700, 1536, 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_ipc_rank_rows, args=(r, world, port, func, m, n, fills, q)) for r in range(world)]
    for p in procs:
        p.start()
    parts = sorted([q.get(timeout=300) for _ in range(world)])
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert parts[0][1] == 0 and parts[-1][2] == n
    assert all(parts[i][2] == parts[i + 1][1] for i in range(world - 1))
    for k in range(fills):
        g = (inputs.gen_costs if func == "minpath3" else inputs.gen_init)(2000 + 17 * k, m, n)
        ref = oracle.minpath3(g) if func == "minpath3" else oracle.min2plus(g, 1)
        last = np.zeros(n, np.int32)
        for rank, c0, c1, res in parts:
            last[c0:c1] = res[k][1]
            assert res[k][0] == (last[c0:c1].min() if c1 > c0 else -7)
        np.testing.assert_array_equal(last, ref.last_row)
        assert min(r[3][k][0] for r in parts if r[2] > r[1]) == ref.score
