"""CPU (gloo) test of the multi-GPU column-strip decomposition used by lddp_fill_multi.

Each process plays one rank: it owns the columns liblddp.so assigns it (lddp_multi_partition,
a host-only call of the C ABI), walks bottom-aligned row strips of the lcs16 height (384 rows =
64 virtual lanes x 6 rows), receives rank g-1's right column for each strip (torch.distributed
recv: the NVLink window store of the GPU path) and sends its own right column to rank g+1 once
the strip is done -- the one-way message order of the kernels (Table II anti-diagonal row,
[L265-L274]).  The assembled last row / score must equal the monolithic oracle."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

STRIP_ROWS = 64 * 6


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _strips(m):
    S = (m + STRIP_ROWS - 1) // STRIP_ROWS
    row0 = m - S * STRIP_ROWS
    return [(max(row0 + s * STRIP_ROWS, 0), row0 + (s + 1) * STRIP_ROWS) for s in range(S)]


def _fill_block(a, b, top, left, corner):
    """LCS cells of a block given the row above (top), the column to the left (left) and the
    corner above-left: the textbook recurrence, row by row (test-side decomposition helper)."""
    rows, cols = len(a), len(b)
    out = np.zeros((rows, cols), np.int64)
    prev = np.concatenate([[corner], top])
    for i in range(rows):
        cur = np.empty(cols + 1, np.int64)
        cur[0] = left[i]
        for j in range(cols):
            cur[j + 1] = prev[j] + 1 if a[i] == b[j] else max(prev[j + 1], cur[j])
        out[i] = cur[1:]
        prev = cur
    return out


def _rank_main(rank, world, port, m, n, seed, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_kumark15_b200 import inputs, lddp
    a, b = inputs.gen_strings(seed, m, n)
    c0, c1 = lddp.lddp_multi_partition(n, world, rank)
    top = np.zeros(c1 - c0, np.int64)          # table row 0 (LCS initialisation)
    last_left_bottom = 0                       # corner for the next strip (rank g-1's value)
    for (r0, r1) in _strips(m):
        rows = r1 - r0
        if rank > 0:
            col = torch.zeros(rows, dtype=torch.int64)
            dist.recv(col, src=rank - 1)       # rank g-1's right column of this strip
            left = col.numpy()
        else:
            left = np.zeros(rows, np.int64)
        corner = last_left_bottom
        blk = _fill_block(a[r0:r1], b[c0:c1], top, left, corner)
        if rank + 1 < world:
            dist.send(torch.from_numpy(np.ascontiguousarray(blk[:, -1])), dst=rank + 1)
        top = blk[-1]
        last_left_bottom = left[-1]
    q.put((rank, c0, top.tolist()))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_column_strip_decomposition_gloo(world):
    import oracle
    from paper_conf_ipps_kumark15_b200 import inputs
    m, n, seed = 1300, 211, 5
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank_main, args=(r, world, port, m, n, seed, q)) for r in range(world)]
    for p in procs:
        p.start()
    parts = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    last = np.zeros(n, np.int64)
    for rank, c0, row in parts:
        last[c0:c0 + len(row)] = row
    a, b = inputs.gen_strings(seed, m, n)
    ref = oracle.lcs(a, b)
    np.testing.assert_array_equal(last, ref.last_row)
    assert last[-1] == ref.score


def test_library_partition():
    """lddp_multi_partition (the C library's rank ranges, used by lddp_fill_multi): contiguous,
    non-empty for cols >= P, covering [0, n) exactly, sizes differing by at most one."""
    from paper_conf_ipps_kumark15_b200 import lddp
    for n in (1, 7, 100, 1000, 100000, 99991):
        for P in (1, 2, 3, 4, 8):
            if n < P:
                continue
            parts = [lddp.lddp_multi_partition(n, P, g) for g in range(P)]
            assert parts[0][0] == 0 and parts[-1][1] == n
            assert all(parts[g][1] == parts[g + 1][0] for g in range(P - 1))
            sizes = [c1 - c0 for c0, c1 in parts]
            assert min(sizes) >= 1 and max(sizes) - min(sizes) <= 1
    with pytest.raises(lddp.LddpError):
        lddp.lddp_multi_partition(10, 2, 2)
