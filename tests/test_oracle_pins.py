"""Pins for the CPU oracle (oracle/), independent of the oracle's own code.

Each pin is something the paper or the mathematics fixes: brute force on tiny inputs, textbook
worked examples (tests/golden/, each cited), closed forms, invariants and special cases.  A
plausible mistake in the oracle (dropped term, wrong sign / index, transposed operand, FMA
contraction) fails at least one of them.  CPU only (no GPU marker).
"""
import itertools

import numpy as np
import pytest

from conftest import golden
from paper_conf_ipps_kumark15_b200 import inputs

# ----------------------------------------------------------------------------------- LCS


def _is_subseq(s, t):
    it = iter(t)
    return all(ch in it for ch in s)


def lcs_brute(a, b):
    """Longest common subsequence by enumerating every subsequence of a (2^m)."""
    m = len(a)
    best = 0
    for mask in range(1 << m):
        k = bin(mask).count("1")
        if k <= best:
            continue
        s = [a[i] for i in range(m) if mask >> i & 1]
        if _is_subseq(s, b):
            best = k
    return best


def test_lcs_brute_force(oracle_mod):
    rng = np.random.default_rng(1234)
    for _ in range(150):
        m, n = rng.integers(0, 10, 2)
        a, b = inputs.gen_strings(int(rng.integers(1 << 30)), int(m), int(n))
        assert oracle_mod.lcs(a, b).score == lcs_brute(list(a), list(b))


def test_lcs_textbook_examples(oracle_mod):
    for case in golden("lcs_examples.json")["cases"]:
        a = np.frombuffer(case["a"].encode(), np.uint8)
        b = np.frombuffer(case["b"].encode(), np.uint8)
        assert oracle_mod.lcs(a, b).score == case["lcs"], case["cite"]


def lcs_scan_rows(a, b):
    """Second, independent formulation: each row is a prefix-max scan (exact in integers):
    L[i][.] = cummax(max(L[i-1][j], L[i-1][j-1] + [a_i == b_j]))."""
    n = len(b)
    prev = np.zeros(n + 1, np.int64)
    rows = []
    for ch in a:
        eq = (b == ch).astype(np.int64)
        cand = np.maximum(prev[1:], prev[:-1] + eq)
        cur = np.concatenate([[0], np.maximum.accumulate(cand)])
        rows.append(cur[1:])
        prev = cur
    return np.array(rows).reshape(len(a), n)


def test_lcs_full_table_vs_scan(oracle_mod):
    for seed, (m, n) in enumerate([(1, 1), (7, 13), (64, 33), (200, 311)]):
        a, b = inputs.gen_strings(seed, m, n)
        r = oracle_mod.lcs(a, b, table=True)
        ref = lcs_scan_rows(a, b)
        np.testing.assert_array_equal(r.table, ref)
        np.testing.assert_array_equal(r.last_row, ref[-1])
        np.testing.assert_array_equal(r.last_col, ref[:, -1])
        assert r.score == ref[-1, -1]


def test_lcs_invariants(oracle_mod):
    a, b = inputs.gen_strings(7, 300, 257)
    s = oracle_mod.lcs(a, b).score
    assert s <= min(len(a), len(b))
    assert oracle_mod.lcs(a, a).score == len(a)
    assert oracle_mod.lcs(b, a).score == s                       # symmetry
    assert oracle_mod.lcs(a, b[:0]).score == 0
    assert oracle_mod.lcs(a, np.frombuffer(b"XYZ" * 9, np.uint8)).score == 0   # disjoint
    assert oracle_mod.lcs(a[:-1], b).score in (s, s - 1)          # appending grows by <= 1
    # Chvatal-Sankoff: for uniform 4-ary strings LCS/n ~ 0.654 (statistical sanity only)
    a, b = inputs.gen_strings(0, 4096, 4096)
    assert 0.60 < oracle_mod.lcs(a, b).score / 4096 < 0.68


# ---------------------------------------------------------------------------- Levenshtein


def lev_bfs(a, b, alphabet):
    """Edit distance by breadth-first search over all strings reachable by unit edits."""
    a, b = tuple(a), tuple(b)
    if a == b:
        return 0
    frontier, seen, d = {a}, {a}, 0
    maxlen = max(len(a), len(b)) + 1
    while True:
        d += 1
        nxt = set()
        for s in frontier:
            cands = []
            for i in range(len(s)):
                cands.append(s[:i] + s[i + 1:])                   # delete
                for c in alphabet:
                    cands.append(s[:i] + (c,) + s[i + 1:])        # substitute
            for i in range(len(s) + 1):
                if len(s) < maxlen:
                    for c in alphabet:
                        cands.append(s[:i] + (c,) + s[i:])        # insert
            for t in cands:
                if t == b:
                    return d
                if t not in seen:
                    seen.add(t)
                    nxt.add(t)
        frontier = nxt


def test_levenshtein_brute_force(oracle_mod):
    rng = np.random.default_rng(99)
    alpha = b"AC"
    for _ in range(60):
        m, n = rng.integers(0, 5, 2)
        a, b = inputs.gen_strings(int(rng.integers(1 << 30)), int(m), int(n), alphabet=alpha)
        assert oracle_mod.levenshtein(a, b).score == lev_bfs(list(a), list(b), list(alpha))


def test_levenshtein_textbook(oracle_mod):
    for case in golden("levenshtein_examples.json")["cases"]:
        a = np.frombuffer(case["a"].encode(), np.uint8)
        b = np.frombuffer(case["b"].encode(), np.uint8)
        assert oracle_mod.levenshtein(a, b).score == case["dist"], case["cite"]


def test_levenshtein_metric_properties(oracle_mod):
    rng = np.random.default_rng(5)
    for _ in range(20):
        a, b = inputs.gen_strings(int(rng.integers(1 << 30)), 40, 37)
        c, _ = inputs.gen_strings(int(rng.integers(1 << 30)), 45, 1)
        dab = oracle_mod.levenshtein(a, b).score
        assert dab == oracle_mod.levenshtein(b, a).score
        assert abs(len(a) - len(b)) <= dab <= max(len(a), len(b))
        assert dab <= oracle_mod.levenshtein(a, c).score + oracle_mod.levenshtein(c, b).score
        # substitution-free bound: edit distance <= indel distance m + n - 2 LCS
        assert dab <= len(a) + len(b) - 2 * oracle_mod.lcs(a, b).score


def test_levenshtein_boundary_rows(oracle_mod):
    # min(i,j) = 0 -> max(i,j) [L325]; first f-row against an empty-prefix reasoning:
    a = np.frombuffer(b"A", np.uint8)
    b = np.frombuffer(b"CACC", np.uint8)
    r = oracle_mod.levenshtein(a, b, table=True)
    # f(1,j) = j - 1 if 'A' in b[:j] else j
    np.testing.assert_array_equal(r.table[0], [1, 1, 2, 3])


# ----------------------------------------------------------------------------------- DTW


def dtw_brute(x, y):
    """Minimum over every monotone warping path (steps (1,0), (0,1), (1,1)) of the sum of
    |x_i - y_j| along it -- exhaustive enumeration (Delannoy-many paths)."""
    m, n = len(x), len(y)
    best = [np.inf]

    def walk(i, j, acc):
        acc += abs(float(x[i]) - float(y[j]))
        if acc >= best[0]:
            return
        if i == m - 1 and j == n - 1:
            best[0] = acc
            return
        if i + 1 < m:
            walk(i + 1, j, acc)
        if j + 1 < n:
            walk(i, j + 1, acc)
        if i + 1 < m and j + 1 < n:
            walk(i + 1, j + 1, acc)

    walk(0, 0, 0.0)
    return best[0]


def test_dtw_brute_force(oracle_mod):
    rng = np.random.default_rng(77)
    for _ in range(80):
        m, n = rng.integers(1, 7, 2)
        x, y = inputs.gen_int_walks(int(rng.integers(1 << 30)), int(m), int(n))
        assert float(oracle_mod.dtw(x, y).score) == dtw_brute(x, y)   # exact: integer data


def test_dtw_worked_examples(oracle_mod):
    for case in golden("dtw_examples.json")["cases"]:
        assert float(oracle_mod.dtw(case["x"], case["y"]).score) == case["dtw"], case["derivation"]


def test_dtw_invariants(oracle_mod):
    x, y = inputs.gen_walks(3, 200, 170)
    d = oracle_mod.dtw(x, y)
    # symmetry, bit-exact: |a-b| = |b-a| exactly and min commutes
    assert oracle_mod.dtw(y, x).score.tobytes() == d.score.tobytes()
    assert oracle_mod.dtw(x, x).score == 0.0
    assert d.score >= 0.0
    # m = 1: a single path, D = sum_j |x0 - y_j| (integer data: exact)
    xi, yi = inputs.gen_int_walks(4, 1, 50)
    assert float(oracle_mod.dtw(xi, yi).score) == float(np.abs(xi[0] - yi).sum())
    # shift invariance on integer data
    xi, yi = inputs.gen_int_walks(5, 30, 41)
    assert oracle_mod.dtw(xi + 7, yi + 7).score == oracle_mod.dtw(xi, yi).score
    # diagonal path bound for m = n
    xi, yi = inputs.gen_int_walks(6, 40, 40)
    assert oracle_mod.dtw(xi, yi).score <= np.abs(xi - yi).sum()
    # empty series: boundary definition
    assert oracle_mod.dtw(x[:0], y[:0]).score == 0.0
    assert np.isinf(oracle_mod.dtw(x[:0], y).score)


def test_dtw_fp32_vs_fp64(oracle_mod):
    """The binary32 DTW is within the north star's 1e-5 relative of the binary64 value."""
    for seed, n in [(0, 512), (1, 2048)]:
        x, y = inputs.gen_walks(seed, n, n)
        d32 = float(oracle_mod.dtw(x, y).score)
        d64 = oracle_mod.dtw_f64(x.astype(np.float64), y.astype(np.float64))
        assert abs(d32 - d64) <= 1e-5 * abs(d64)


# ------------------------------------------------------------------------------------ FS


def test_fs_worked_examples(oracle_mod):
    for case in golden("fs_examples.json")["cases"]:
        out = oracle_mod.fs(np.array(case["in"], np.uint8))
        np.testing.assert_array_equal(out, np.array(case["out"], np.uint8), err_msg=case["name"])


def test_fs_one_row_and_one_column_reduce_to_1d(oracle_mod):
    """1-row image: v_j = in_j + (7/16) e_{j-1};  1-column image: v_i = in_i + (5/16) e_{i-1}
    (the only surviving diffusion direction), binary32 multiply-then-add."""
    img = inputs.gen_image(8, 1, 500, "uniform")
    for arr, w in [(img[0], np.float32(7 / 16)), (img[0], np.float32(5 / 16))]:
        e, outs = np.float32(0), []
        for p in arr:
            v = np.float32(np.float32(p) + np.float32(e * w))
            o = np.float32(255) if v >= np.float32(128) else np.float32(0)
            outs.append(int(o))
            e = np.float32(v - o)
        shape = (1, len(arr)) if w == np.float32(7 / 16) else (len(arr), 1)
        np.testing.assert_array_equal(oracle_mod.fs(arr.reshape(shape)).ravel(), outs)


def test_fs_invariants(oracle_mod):
    img = inputs.gen_image(11, 97, 131, "ramp")
    out, err = oracle_mod.fs(img, want_err=True)
    assert set(np.unique(out)) <= {0, 255}
    # each pixel: out = v >= 128 ? 255 : 0 and e = v - out  =>  e in [-127, 128) when v in [0,255+]
    assert np.all((out == 255) == (err + out >= 128))
    # intensity conservation: sum(in) - sum(out) = sum of error diffused off the image edges
    H, W = img.shape
    drop = np.zeros((H, W))
    drop[:, -1] += 7 / 16                  # right neighbour missing
    drop[-1, :] += 3 / 16 + 5 / 16 + 1 / 16  # row below missing
    drop[:-1, 0] += 3 / 16                 # down-left missing
    drop[:-1, -1] += 1 / 16                # down-right missing
    lhs = float(img.astype(np.float64).sum() - out.astype(np.float64).sum())
    rhs = float((err.astype(np.float64) * drop).sum())
    assert abs(lhs - rhs) < 1e-3 * H * W
    # statistical: mean preserved (uniform input -> ~50% white)
    u = inputs.gen_image(12, 256, 256, "uniform")
    frac = (oracle_mod.fs(u) == 255).mean()
    assert abs(frac - u.mean() / 255.0) < 0.01


def test_fs_2x2_derivation_intermediates(oracle_mod):
    """Intermediate errors of the hand-worked 2x2 case (tests/golden/fs_examples.json).
    (FMA contraction is caught by the 1-row / 1-column test, whose errors carry many bits.)"""
    img = np.full((2, 2), 100, np.uint8)
    out, err = oracle_mod.fs(img, want_err=True)
    # derivation: e(1,0) = 110.390625 exactly, v(1,1) = 119.7802734375
    assert err[1, 0] == np.float32(110.390625)
    assert err[1, 1] == np.float32(119.7802734375)


# ------------------------------------------------------------------------------ MIN_PATH3


def minpath_brute(c):
    H, W = c.shape
    best = np.full(W, np.iinfo(np.int64).max)
    for j0 in range(W):
        for moves in itertools.product((-1, 0, 1), repeat=H - 1):
            j, s, ok = j0, int(c[0, j0]), True
            for i, mv in enumerate(moves, start=1):
                j += mv
                if not 0 <= j < W:
                    ok = False
                    break
                s += int(c[i, j])
            if ok:
                best[j] = min(best[j], s)
    return best


def test_minpath_brute_force(oracle_mod):
    rng = np.random.default_rng(3)
    for _ in range(40):
        H, W = int(rng.integers(1, 6)), int(rng.integers(1, 6))
        c = inputs.gen_costs(int(rng.integers(1 << 30)), H, W, hi=50)
        r = oracle_mod.minpath3(c)
        ref = minpath_brute(c)
        np.testing.assert_array_equal(r.last_row, ref)
        assert r.score == ref.min()


def test_minpath_worked_example(oracle_mod):
    for case in golden("minpath_examples.json")["cases"]:
        r = oracle_mod.minpath3(np.array(case["cost"], np.int32))
        np.testing.assert_array_equal(r.last_row, case["last_row"])
        assert r.score == case["min"]


def test_minpath_special_cases(oracle_mod):
    c = inputs.gen_costs(9, 50, 1)
    r = oracle_mod.minpath3(c, table=True)
    np.testing.assert_array_equal(r.table[:, 0], np.cumsum(c[:, 0]))     # W = 1: column sum
    k = 13
    r = oracle_mod.minpath3(np.full((20, 17), k, np.int32), table=True)
    np.testing.assert_array_equal(r.table, (np.arange(20)[:, None] + 1) * k * np.ones((1, 17), np.int64))
    # monotone: raising a cost never lowers any f
    c = inputs.gen_costs(10, 30, 30)
    base = oracle_mod.minpath3(c, table=True).table
    c2 = c.copy()
    c2[12, 7] += 100
    assert np.all(oracle_mod.minpath3(c2, table=True).table >= base)


def test_minpath_matches_dijkstra(oracle_mod):
    """Mid-size cross-check: Bellman-Ford relaxation on the layered DAG in numpy."""
    c = inputs.gen_costs(21, 60, 45)
    H, W = c.shape
    dist = c[0].astype(np.int64)
    for i in range(1, H):
        padded = np.concatenate([[np.iinfo(np.int64).max // 4], dist, [np.iinfo(np.int64).max // 4]])
        dist = c[i] + np.minimum(np.minimum(padded[:-2], padded[1:-1]), padded[2:])
    np.testing.assert_array_equal(oracle_mod.minpath3(c).last_row, dist)


# ------------------------------------------------------------------------------ MIN2_PLUS


def test_min2plus_closed_form(oracle_mod):
    """f(i,j) = i*c + min(init[0][max(0, j-i) .. j]) -- a sliding-window min of row 0."""
    rng = np.random.default_rng(17)
    for _ in range(30):
        H, W = int(rng.integers(1, 40)), int(rng.integers(1, 40))
        cst = int(rng.integers(0, 5))
        init = inputs.gen_init(int(rng.integers(1 << 30)), H, W, hi=1000)
        r = oracle_mod.min2plus(init, cst, table=True)
        for i in range(H):
            ref = [i * cst + init[0, max(0, j - i): j + 1].min() for j in range(W)]
            np.testing.assert_array_equal(r.table[i], ref)


def test_min2plus_brute_paths(oracle_mod):
    init = inputs.gen_init(2, 5, 6, hi=100)
    cst = 3
    r = oracle_mod.min2plus(init, cst, table=True)
    H, W = init.shape
    for i in range(H):
        for j in range(W):
            best = None
            for moves in itertools.product((0, 1), repeat=i):    # down or down-right
                j0 = j - sum(moves)
                if j0 >= 0:
                    v = int(init[0, j0]) + i * cst
                    best = v if best is None else min(best, v)
            assert r.table[i, j] == best


# --------------------------------------------------------------------------- DIAG_MAXPLUS


def test_diagmaxplus_closed_form(oracle_mod):
    """f(i,j) = max(max_{k<K} init[i-k][j-k] + (k+1)c, init[i-K][j-K] + K c), K = min(i,j):
    along each diagonal the recurrence unrolls into an offset prefix-max."""
    rng = np.random.default_rng(23)
    for _ in range(30):
        H, W = int(rng.integers(1, 30)), int(rng.integers(1, 30))
        cst = int(rng.integers(0, 4))
        init = inputs.gen_init(int(rng.integers(1 << 30)), H, W, hi=50)
        r = oracle_mod.diagmaxplus(init, cst, table=True)
        for i in range(H):
            for j in range(W):
                K = min(i, j)
                cands = [int(init[i - k, j - k]) + (k + 1) * cst for k in range(K)]
                cands.append(int(init[i - K, j - K]) + K * cst)
                assert r.table[i, j] == max(cands)
        np.testing.assert_array_equal(r.last_row, r.table[-1])
        np.testing.assert_array_equal(r.last_col, r.table[:, -1])


def test_diagmaxplus_constant(oracle_mod):
    r = oracle_mod.diagmaxplus(np.full((9, 11), 5, np.int32), 0, table=True)
    assert np.all(r.table == 5)


# ------------------------------------------------- symmetric twins (Vertical, mInverted-L)


def test_min2plus_v_closed_form(oracle_mod):
    """Vertical twin: f(i,j) = j*c + min(init[max(0, i-j) .. i][0]) -- a sliding-window min of
    column 0 (the transpose of min2plus's closed form)."""
    rng = np.random.default_rng(29)
    for _ in range(30):
        H, W = int(rng.integers(1, 40)), int(rng.integers(1, 40))
        cst = int(rng.integers(0, 5))
        init = inputs.gen_init(int(rng.integers(1 << 30)), H, W, hi=1000)
        r = oracle_mod.min2plus_v(init, cst, table=True)
        for j in range(W):
            ref = [j * cst + init[max(0, i - j): i + 1, 0].min() for i in range(H)]
            np.testing.assert_array_equal(r.table[:, j], ref)
        np.testing.assert_array_equal(r.last_col, r.table[:, -1])
        assert r.score == r.table[:, -1].min()


def test_min2plus_v_brute_paths(oracle_mod):
    """f(i,j) = min over monotone paths of right / up-right moves from column 0 to (i, j)."""
    init = inputs.gen_init(3, 6, 5, hi=100)
    cst = 2
    r = oracle_mod.min2plus_v(init, cst, table=True)
    H, W = init.shape
    for i in range(H):
        for j in range(W):
            best = None
            for moves in itertools.product((0, 1), repeat=j):    # right (L) or down-right (UL)
                i0 = i - sum(moves)
                if i0 >= 0:
                    v = int(init[i0, 0]) + j * cst
                    best = v if best is None else min(best, v)
            assert r.table[i, j] == best


def test_antidiag_maxplus_closed_form(oracle_mod):
    """mInverted-L twin: along each anti-diagonal chain (i-k, j+k) the recurrence unrolls into an
    offset prefix-max: f(i,j) = max(max_{k<K} init[i-k][j+k] + (k+1)c, init[i-K][j+K] + K c),
    K = min(i, W-1-j)."""
    rng = np.random.default_rng(31)
    for _ in range(30):
        H, W = int(rng.integers(1, 30)), int(rng.integers(1, 30))
        cst = int(rng.integers(0, 4))
        init = inputs.gen_init(int(rng.integers(1 << 30)), H, W, hi=50)
        r = oracle_mod.antidiag_maxplus(init, cst, table=True)
        for i in range(H):
            for j in range(W):
                K = min(i, W - 1 - j)
                cands = [int(init[i - k, j + k]) + (k + 1) * cst for k in range(K)]
                cands.append(int(init[i - K, j + K]) + K * cst)
                assert r.table[i, j] == max(cands)
        np.testing.assert_array_equal(r.last_row, r.table[-1])
        np.testing.assert_array_equal(r.last_col, r.table[:, 0])


def test_twins_are_transpose_and_mirror(oracle_mod):
    """[L111]: Vertical = transpose of Horizontal, mInverted-L = mirror of Inverted-L.  The twin
    oracles equal the transposed / mirrored runs of the (separately pinned) originals."""
    rng = np.random.default_rng(37)
    for _ in range(10):
        H, W = int(rng.integers(1, 50)), int(rng.integers(1, 50))
        init = inputs.gen_init(int(rng.integers(1 << 30)), H, W, hi=1 << 20)
        v = oracle_mod.min2plus_v(init, 3, table=True)
        h = oracle_mod.min2plus(np.ascontiguousarray(init.T), 3, table=True)
        np.testing.assert_array_equal(v.table, h.table.T)
        a = oracle_mod.antidiag_maxplus(init, 2, table=True)
        d = oracle_mod.diagmaxplus(np.ascontiguousarray(init[:, ::-1]), 2, table=True)
        np.testing.assert_array_equal(a.table, d.table[:, ::-1])


# -------------------------------------------------------------------- Table I / Fig. 2


SCHEDULES = {
    # 0-based iteration number t(i, j) of every pattern of Fig. 2 [L117-L122] on an H x W grid
    "Anti-diagonal": lambda i, j, H, W: i + j,
    "Horizontal": lambda i, j, H, W: i,
    "Inverted-L": lambda i, j, H, W: min(i, j),
    "Knight-Move": lambda i, j, H, W: 2 * i + j,
    "Vertical": lambda i, j, H, W: j,
    "mInverted-L": lambda i, j, H, W: min(i, W - 1 - j),
}
OFFSETS = {"L": (0, -1), "UL": (-1, -1), "U": (-1, 0), "UR": (-1, 1)}   # RS(i,j) [L90]


def schedule_valid(pattern, mask, H=7, W=7):
    t = SCHEDULES[pattern]
    for i in range(H):
        for j in range(W):
            for nb in mask:
                di, dj = OFFSETS[nb]
                ii, jj = i + di, j + dj
                if 0 <= ii < H and 0 <= jj < W and not t(ii, jj, H, W) < t(i, j, H, W):
                    return False
    return True


def test_table1_patterns_order_every_dependency():
    """Mechanical check of Table I against the Fig. 2 schedules: the pattern the paper assigns
    to each contributing set strictly orders every dependency; Knight-Move covers all 15."""
    rows = golden("table1.json")["rows"]
    assert len(rows) == 15
    for row in rows:
        mask = [k for k in ("L", "UL", "U", "UR") if row[k] == "Y"]
        assert schedule_valid(row["pattern"], mask), row
        assert schedule_valid("Knight-Move", mask), row


def test_fig2_knight_grid():
    fig = golden("fig2_knight.json")
    grid = np.array(fig["grid"])
    H, W = grid.shape
    ref = np.array([[SCHEDULES["Knight-Move"](i, j, H, W) + 1 for j in range(W)] for i in range(H)])
    np.testing.assert_array_equal(grid, ref)
    counts = fig["iterations_6x6"]
    for pat, key in [("Anti-diagonal", "anti_diagonal"), ("Horizontal", "horizontal"),
                     ("Inverted-L", "inverted_l"), ("Knight-Move", "knight_move"),
                     ("Vertical", "vertical")]:
        vals = {SCHEDULES[pat](i, j, 6, 6) for i in range(6) for j in range(6)}
        assert len(vals) == counts[key], pat


# ---------------------------------------------------------------------------------- traceback
# Reading R14: the traceback rule of each sequence f.  Pinned by the textbook LCS
# (CLRS Fig. 15.8 prints "BCBA" for X = ABCBDAB, Y = BDCABA with the up-on-ties rule) and by
# properties any valid alignment must have, checked without the traceback code.

def _is_subsequence(s, t):
    it = iter(t)
    return all(c in it for c in s)


def _moves_ok(path, m, n):
    if not path or path[0] != (m, n):
        return False
    for (i0, j0), (i1, j1) in zip(path, path[1:]):
        if (i0 - i1, j0 - j1) not in ((1, 1), (1, 0), (0, 1)):
            return False
    return True


def test_traceback_lcs_textbook(oracle_mod):
    a, b = np.frombuffer(b"ABCBDAB", np.uint8), np.frombuffer(b"BDCABA", np.uint8)
    r = oracle_mod.lcs(a, b, table=True)
    path = oracle_mod.traceback("lcs", a, b, r.table)
    assert oracle_mod.lcs_string(a, b, path) == b"BCBA"


def test_traceback_lcs_random(oracle_mod):
    rng = np.random.default_rng(3)
    for _ in range(60):
        m, n = rng.integers(1, 40, 2)
        a = rng.integers(65, 69, m).astype(np.uint8)
        b = rng.integers(65, 69, n).astype(np.uint8)
        r = oracle_mod.lcs(a, b, table=True)
        path = oracle_mod.traceback("lcs", a, b, r.table)
        s = oracle_mod.lcs_string(a, b, path)
        assert _moves_ok(path, m, n)
        assert len(s) == r.score
        assert _is_subsequence(s, bytes(a)) and _is_subsequence(s, bytes(b))


def test_traceback_dtw_path_cost(oracle_mod):
    """Integer-valued series: the path's summed |x - y| equals D(m, n) exactly; the path is a
    warping path from (m, n) to (1, 1)."""
    rng = np.random.default_rng(4)
    for _ in range(60):
        m, n = rng.integers(1, 30, 2)
        x = rng.integers(-20, 21, m).astype(np.float32)
        y = rng.integers(-20, 21, n).astype(np.float32)
        r = oracle_mod.dtw(x, y, table=True)
        path = oracle_mod.traceback("dtw", x, y, r.table)
        assert _moves_ok(path, m, n) and path[-1] == (1, 1)
        assert sum(abs(float(x[i - 1]) - float(y[j - 1])) for i, j in path) == float(r.score)


def test_traceback_levenshtein_cost(oracle_mod):
    """The alignment the path describes (diagonal: 0 / 1, vertical / horizontal: 1, then the
    boundary tail) costs exactly the distance."""
    rng = np.random.default_rng(5)
    for _ in range(60):
        m, n = rng.integers(1, 30, 2)
        a = rng.integers(65, 69, m).astype(np.uint8)
        b = rng.integers(65, 69, n).astype(np.uint8)
        r = oracle_mod.levenshtein(a, b, table=True)
        path = oracle_mod.traceback("levenshtein", a, b, r.table)
        assert _moves_ok(path, m, n)
        cost = 0
        for k, (i, j) in enumerate(path):
            if k + 1 < len(path):
                i1, j1 = path[k + 1]
            else:   # the move that leaves the table interior
                i1, j1 = i - 1, j - 1
                if not (i >= 1 and j >= 1):
                    break
                here = r.table[i - 1][j - 1]
                diag = (max(i - 1, j - 1) if (i == 1 or j == 1) else r.table[i - 2][j - 2])
                if not ((a[i - 1] == b[j - 1] and here == diag) or here == diag + 1):
                    up = max(i - 1, j) if i == 1 else r.table[i - 2][j - 1]
                    i1, j1 = (i - 1, j) if here == up + 1 else (i, j - 1)
            cost += (int(a[i - 1] != b[j - 1]) if (i - i1, j - j1) == (1, 1) else 1)
            if k + 1 == len(path):
                cost += max(i1, j1)   # boundary tail: pure deletions / insertions
        assert cost == r.score
