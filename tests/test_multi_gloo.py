"""CPU (gloo) test of the multi-GPU column-strip decomposition used by lddp_fill_multi.

Each process plays one rank: it owns columns [floor(g*n/P), floor((g+1)*n/P)), walks the same
bottom-aligned row strips as the wavefront kernel (512 rows = 4 warps x 32 lanes x 4 rows),
receives rank g-1's right column for each strip (torch.distributed recv: the NVLink window
write of the GPU path) and sends its own right column to rank g+1 once the strip is done --
the same one-way message order as the kernel (Table II anti-diagonal row, [L265-L274]).  The
assembled last row / score must equal the monolithic oracle."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

STRIP_ROWS = 4 * 32 * 4


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
    from paper_conf_ipps_kumark15_b200 import inputs
    a, b = inputs.gen_strings(seed, m, n)
    c0, c1 = rank * n // world, (rank + 1) * n // world
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


def test_partition_matches_library_formula():
    """The C library's rank ranges: floor(g*n/P) .. floor((g+1)*n/P) cover [0, n) exactly."""
    for n in (1, 7, 100, 100000, 99991):
        for P in (1, 2, 3, 4, 8):
            if n < P:
                continue
            edges = [g * n // P for g in range(P + 1)]
            assert edges[0] == 0 and edges[-1] == n
            assert all(edges[g + 1] > edges[g] for g in range(P))
