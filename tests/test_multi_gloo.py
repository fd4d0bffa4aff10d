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


# ------------------------------------------------- prev-row: two-way trapezoid halos over gloo
HB = 32          # band height = halo width of the column-block kernel's default geometry
BW = 64          # its own columns per block: strips are whole blocks
GARBAGE = -(1 << 40)   # value of a halo cell whose inputs are stale (must never reach own columns)


def _rows_rank_main(rank, world, port, m, n, seed, q):
    """Rank g owns whole BW-column blocks; every band of HB rows it computes its columns plus HB
    halo columns each side from the halo values exchanged at the band start (one send + one recv
    per side and band: Table II case 2 two-way halo [L265-L274], [L193-L195]).  Cells are the
    min-path recurrence c + min(UL, U, UR) [L298]; a halo cell whose left / right input lies
    outside the extended window takes GARBAGE, so a too-narrow halo would corrupt own columns."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_kumark15_b200 import inputs
    cost = inputs.gen_costs(seed, m, n).astype(np.int64)
    NB = (n + BW - 1) // BW
    c0 = min(rank * NB // world * BW, n)
    c1 = min((rank + 1) * NB // world * BW, n)
    big = np.int64(1 << 50)                       # out-of-table neighbour (f's boundary)
    lo, hi = c0 - HB, c1 + HB                     # extended window [lo, hi)
    cols = np.arange(lo, hi)
    inside = (cols >= 0) & (cols < n)
    cur = np.where(inside, 0, big).astype(np.int64)   # row -1: top initialisation
    for r0 in range(0, m, HB):
        nr = min(HB, m - r0)
        for i in range(r0, r0 + nr):
            ul = np.concatenate([[GARBAGE], cur[:-1]])
            ur = np.concatenate([cur[1:], [GARBAGE]])
            ul[0] = big if lo - 1 < 0 else GARBAGE
            ur[-1] = big if hi >= n else GARBAGE
            c = np.where(inside, cost[i, np.clip(cols, 0, n - 1)], 0)
            nxt = c + np.minimum(np.minimum(ul, cur), ur)
            cur = np.where(inside, nxt, big)
        if r0 + HB >= m:
            break
        # band boundary: own edges out, neighbours' edges in (both directions)
        reqs = []
        if rank > 0:
            reqs.append(dist.isend(torch.from_numpy(cur[HB:2 * HB].copy()), dst=rank - 1))
        if rank + 1 < world:
            reqs.append(dist.isend(torch.from_numpy(cur[-2 * HB:-HB].copy()), dst=rank + 1))
        if rank > 0:
            t = torch.zeros(HB, dtype=torch.int64)
            dist.recv(t, src=rank - 1)
            cur[:HB] = t.numpy()
        if rank + 1 < world:
            t = torch.zeros(HB, dtype=torch.int64)
            dist.recv(t, src=rank + 1)
            cur[-HB:] = t.numpy()
        for rq in reqs:
            rq.wait()
    own = cur[HB:HB + (c1 - c0)]
    q.put((rank, c0, c1, own.tolist()))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_prev_row_two_way_halo_gloo(world):
    import oracle
    from paper_conf_ipps_kumark15_b200 import inputs
    m, n, seed = 301, 448, 9
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rows_rank_main, args=(r, world, port, m, n, seed, q)) for r in range(world)]
    for p in procs:
        p.start()
    parts = sorted(q.get(timeout=240) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert parts[0][1] == 0 and parts[-1][2] == n
    last = np.zeros(n, np.int64)
    for rank, c0, c1, row in parts:
        assert c0 % BW == 0
        last[c0:c1] = row
    ref = oracle.minpath3(inputs.gen_costs(seed, m, n))
    np.testing.assert_array_equal(last, ref.last_row)
    assert last.min() == ref.score
