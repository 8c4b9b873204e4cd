"""Pins for the CPU oracle (oracle/oracle.c) against things other than itself.

Each test names the passage or the mathematical fact it pins.  Together they are
chosen so that a plausible mistake in any oracle function (a dropped term, a wrong
sign or index, an off-by-one in a coordinate, a swapped tie-break, a transposed
operand) fails at least one of them.  CPU only.
"""
import json
import os

import numpy as np
import pytest

import graphgen as G
import oracle as O

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def rand_graph(rs, m, n, max_len, dup=False, seed=0, vals="int"):
    kind = rs.randint(4)
    if kind == 0:
        rl = rs.randint(0, max_len + 1, size=m)
    elif kind == 1:   # many empty rows
        rl = np.where(rs.rand(m) < 0.6, 0, rs.randint(0, max_len + 1, size=m))
    elif kind == 2:   # one long row somewhere
        rl = rs.randint(0, 3, size=m)
        if m:
            rl[rs.randint(m)] = max_len * 4
    else:
        rl = rs.randint(0, max_len + 1, size=m)
        if m:
            rl[0] = max_len * 3
            rl[-1] = max_len * 3
    return G.random_csr(m, n, rl.astype(np.int32), seed, canonical=not dup, values=vals)


def merrill_search(rp, d):
    """Merrill & Garland [18] MergePathSearch (ref. cited at P:31): list A is
    the row-end offsets RP[1..m], list B the natural numbers 0..nnz-1; A[i] <= B[j]
    consumes A first.  Returns (x, y) with x + y = d.  Textbook formulation."""
    m, nnz = len(rp) - 1, int(rp[-1])
    lo, hi = max(0, d - nnz), min(d, m)
    while lo < hi:
        pivot = (lo + hi) // 2
        if rp[1 + pivot] <= d - pivot - 1:
            lo = pivot + 1
        else:
            hi = pivot
    return lo, d - lo


# --------------------------------------------------------------------------------
# O1 / O2 / O3: the row-wise product
# --------------------------------------------------------------------------------
def test_o1_equals_dense_bruteforce_integer_exact():
    rs = np.random.RandomState(1)
    for trial in range(60):
        m, n = rs.randint(0, 40), rs.randint(1, 40)
        g = rand_graph(rs, m, n, 6, dup=bool(trial % 2), seed=trial)
        K = int(rs.randint(1, 9))
        B = G.dense_int(n, K, seed=trial)
        C1 = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        C3 = O.dense_spmm_f64(g.row_ptr, g.col_idx, g.val, n, B)
        assert np.array_equal(C1, C3)


def test_o1_equals_dense_bruteforce_float():
    rs = np.random.RandomState(2)
    for trial in range(30):
        m, n = rs.randint(1, 60), rs.randint(1, 60)
        g = rand_graph(rs, m, n, 8, dup=True, seed=100 + trial, vals="int")
        g.val = (rs.rand(g.nnz).astype(np.float32) - 0.5)
        B = G.dense_uniform(n, 5, seed=trial)
        C1 = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        C3 = O.dense_spmm_f64(g.row_ptr, g.col_idx, g.val, n, B)
        np.testing.assert_allclose(C1, C3, rtol=1e-12, atol=1e-14)


def test_o1_identity_gives_B():
    n, K = 257, 7
    rp = np.arange(n + 1, dtype=np.int32)
    ci = np.arange(n, dtype=np.int32)
    val = np.ones(n, np.float32)
    B = G.dense_uniform(n, K, seed=3)
    C = O.csr_spmm_f64(rp, ci, val, B, want_bound=False)
    assert np.array_equal(C, B.astype(np.float64))


def test_o1_ones_gives_weighted_degree():
    g = G.workload("cora")
    B = np.ones((g.n, 4), np.float32)
    C = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
    rows = np.repeat(np.arange(g.m), np.diff(g.row_ptr))
    wdeg = np.bincount(rows, weights=g.val.astype(np.float64), minlength=g.m)
    for k in range(4):
        np.testing.assert_allclose(C[:, k], wdeg, rtol=1e-13, atol=0)
    assert np.all(C[np.diff(g.row_ptr) == 0] == 0.0)


def test_o1_linear_in_B_and_bound():
    rs = np.random.RandomState(4)
    g = rand_graph(rs, 80, 50, 9, seed=5)
    g.val = rs.randn(g.nnz).astype(np.float32)
    B1 = G.dense_int(50, 6, seed=1)      # integer B: 2*B1 - 3*B2 is exact in fp32
    B2 = G.dense_int(50, 6, seed=2)
    C1, b1 = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B1)
    C2, _ = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B2)
    C3, _ = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, 2 * B1 - 3 * B2)
    np.testing.assert_allclose(C3, 2 * C1 - 3 * C2, rtol=1e-12, atol=1e-12)
    assert np.all(b1 >= np.abs(C1) - 1e-15)
    # |A|,|B| >= 0 makes the bound equal to the product
    Cp, bp = O.csr_spmm_f64(g.row_ptr, g.col_idx, np.abs(g.val), np.abs(B1))
    np.testing.assert_allclose(bp, Cp, rtol=1e-15)


def test_o1_row_subset_matches_full():
    g = G.workload("pubmed")
    B = G.features("pubmed", 16)
    full = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
    rows = np.array([0, 5, g.m - 1, 17, 5], np.int64)
    sub = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, rows=rows, want_bound=False)
    assert np.array_equal(sub, full[rows])


def test_check_tolerance_o8():
    ref = np.array([[1.0, -2.0]])
    bnd = np.array([[1.0, 2.0]])
    assert O.check(ref + 0.5e-5, ref, bnd)["ok"]
    r = O.check(ref + np.array([[0.0, 3e-5]]), ref, bnd)
    assert not r["ok"] and r["violations"] == 1
    r = O.check(np.array([[np.nan, -2.0]]), ref, bnd)
    assert not r["ok"] and r["nonfinite"] == 1


# --------------------------------------------------------------------------------
# O4 / O5: merge-path coordinates (Alg. 1)
# --------------------------------------------------------------------------------
def test_o4_closed_form_equals_walk_and_merrill():
    rs = np.random.RandomState(5)
    for trial in range(400):
        m, n = rs.randint(0, 13), 12
        g = rand_graph(rs, m, n, 5, seed=trial)
        rp = g.row_ptr
        xs, ys = O.merge_walk(rp)
        M = g.m + g.nnz
        assert xs[M] == g.m and ys[M] == g.nnz
        for d in range(M + 1):
            x, y = O.merge_coord(rp, d)
            assert (x, y) == (xs[d], ys[d])
            assert (x, y) == merrill_search(list(rp), d)
            # the unique point on the diagonal with RP[x] <= y <= RP[x+1] (reading R5)
            valid = [xx for xx in range(max(0, d - g.nnz), min(d, g.m) + 1)
                     if rp[xx] <= d - xx and (xx == g.m or d - xx <= rp[xx + 1])]
            assert valid == [x]


def test_o5_walk_steps_are_unit():
    rs = np.random.RandomState(6)
    g = rand_graph(rs, 30, 30, 6, seed=9)
    xs, ys = O.merge_walk(g.row_ptr)
    dx, dy = np.diff(xs), np.diff(ys)
    assert np.all(dx + dy == 1) and np.all(dx >= 0) and np.all(dy >= 0)
    # a row end is taken exactly when all its non-zeros are consumed
    for d in range(len(dx)):
        if dx[d] == 1:
            assert g.row_ptr[xs[d] + 1] <= ys[d]


@pytest.mark.parametrize("completion", [
    [13, 14, 15, 15, 16, 16, 16, 16],
    [12, 12, 12, 12, 12, 12, 12, 16],
    [16, 16, 16, 16, 16, 16, 16, 16],
    [13, 13, 14, 14, 15, 15, 16, 16],
])
def test_fig3_example(completion):
    with open(os.path.join(GOLD, "fig3.json")) as f:
        fx = json.load(f)
    rp = np.array(fx["row_ptr_prefix"] + completion, np.int32)
    assert len(rp) == fx["rows"] + 1 and rp[-1] == fx["nnz"]
    M = fx["rows"] + fx["nnz"]
    assert M == fx["merge_items"]
    P, L = O.plan(fx["rows"], fx["nnz"], cost=fx["items_per_thread"], min_parts=1)
    assert (P, L) == (fx["threads"], fx["items_per_thread"])
    # Alg. 1 line 3 as printed agrees with reading R1 here (P does not divide M)
    assert (M + P) // P == L
    cx, cy = O.partition(rp, P, L)
    d = (cx + cy).tolist()
    assert d[:-1] == fx["start_costs"]
    assert d[1:] == fx["end_costs_reading_R3"]
    # thread 2 (p = 1): paper coordinates (1,6) and (3,11) = (x+1, y-1)
    assert (int(cx[1]) + 1, int(cy[1]) - 1) == tuple(fx["thread2_start_paper"])
    assert (int(cx[2]) + 1, int(cy[2]) - 1) == tuple(fx["thread2_end_paper"])
    assert int(cx[2] - cx[1]) == fx["thread2_rows"]
    assert (int(cy[1]), int(cy[2]) - 1) == (fx["thread2_nnz_first"], fx["thread2_nnz_last"])
    assert (cy[1] != rp[cx[1]]) == fx["thread2_start_partial"]
    assert (cy[2] != rp[cx[2]]) == fx["thread2_end_partial"]
    assert tuple(cx[[0, 4]]) == (0, 10) and tuple(cy[[0, 4]]) == (0, 16)


def test_plan_properties():
    for (m, nnz, cost, pmin) in [(0, 0, 5, 1), (10, 16, 7, 1), (10, 16, 7, 1024), (5, 0, 2, 1),
                                 (232965, 114615892, 256, 7104), (3, 100, 1000, 1),
                                 (26, 0, 13, 2), (10, 16, 13, 2)]:
        P, L = O.plan(m, nnz, cost, pmin)
        M = m + nnz
        assert P == max(-(-M // cost), pmin)
        assert P * L >= M and (L == 0 or (P * L - M) < P)
    # printed Alg. 1 line 3 differs from reading R1 when P divides M (G1)
    assert O.plan(10, 16, 13, 2) == (2, 13)
    with pytest.raises(ValueError):
        O.plan(1, 1, 0, 1)


def test_o4_partition_invariants():
    rs = np.random.RandomState(7)
    for trial in range(120):
        g = rand_graph(rs, rs.randint(0, 200), 50, 12, seed=trial)
        M = g.m + g.nnz
        P = int(rs.randint(1, 40))
        L = -(-M // P)
        cx, cy = O.partition(g.row_ptr, P, L)
        rp = g.row_ptr
        assert cx[0] == 0 and cy[0] == 0 and cx[P] == g.m and cy[P] == g.nnz
        d = cx.astype(np.int64) + cy
        assert np.array_equal(d, np.minimum(np.arange(P + 1) * L, M))
        assert np.all(np.diff(cx) >= 0) and np.all(np.diff(cy) >= 0)
        for p in range(P + 1):
            assert rp[cx[p]] <= cy[p]
            if cx[p] < g.m:
                assert cy[p] <= rp[cx[p] + 1]
        items = np.diff(d)
        assert np.array_equal(items, np.minimum(L, np.maximum(0, M - np.arange(P) * L)))
        assert items.sum() == M


def test_o4_sub_range_diagonals():
    rs = np.random.RandomState(8)
    g = rand_graph(rs, 100, 60, 10, seed=3)
    M = g.m + g.nnz
    b, e = M // 3, 2 * M // 3
    cx, cy = O.partition(g.row_ptr, 7, -(-(e - b) // 7), b, e)
    xs, ys = O.merge_walk(g.row_ptr)
    dd = cx.astype(np.int64) + cy
    assert dd[0] == b and dd[-1] == e
    assert np.array_equal(cx, xs[dd]) and np.array_equal(cy, ys[dd])


def test_o4_partition64_small_equals_int32_partition():
    """NEXT-4: the int64-offset partition is the same Alg. 1 closed form."""
    rs = np.random.RandomState(17)
    for trial in range(60):
        g = rand_graph(rs, rs.randint(0, 150), 40, 10, seed=trial)
        M = g.m + g.nnz
        P = int(rs.randint(1, 30))
        L = -(-M // P)
        cx, cy = O.partition(g.row_ptr, P, L)
        cx64, cy64 = O.partition64(g.row_ptr.astype(np.int64), P, L)
        assert cy64.dtype == np.int64
        assert np.array_equal(cx, cx64) and np.array_equal(cy.astype(np.int64), cy64)


def test_o4_partition64_beyond_2p31_matches_searchsorted():
    """NEXT-4: m + nnz > 2^31.  x_p = max{x : x + RP[x] <= d_p} (reading R4) computed by
    numpy's searchsorted over the strictly increasing s(x) = x + RP[x] -- a library
    primitive, not the oracle's bisection -- and the unique-point property
    RP[x] <= y <= RP[x+1] (reading R5), including diagonals at the 2^31 boundary."""
    rs = np.random.RandomState(18)
    m = 200_000
    rl = rs.randint(0, 40_000, size=m).astype(np.int64)
    rl[rs.randint(m, size=5)] = 3_000_000_000 // 5   # a few rows past 2^31 on their own
    rl[rl % 7 == 0] = 0
    rp = np.zeros(m + 1, np.int64)
    np.cumsum(rl, out=rp[1:])
    nnz = int(rp[-1])
    assert m + nnz > 2 ** 32
    s = np.arange(m + 1, dtype=np.int64) + rp
    P = 5000
    L = -(-(m + nnz) // P)
    cx, cy = O.partition64(rp, P, L)
    d = np.minimum(np.arange(P + 1, dtype=np.int64) * L, m + nnz)
    x_ref = np.searchsorted(s, d, side="right") - 1
    assert np.array_equal(cx.astype(np.int64), x_ref)
    assert np.array_equal(cy, d - x_ref)
    assert np.all(rp[cx] <= cy)
    inner = cx < m
    assert np.all(cy[inner] <= rp[cx[inner] + 1])
    # single diagonals straddling 2^31 (through the sub-range form of line 4)
    for dd in (2 ** 31 - 1, 2 ** 31, 2 ** 31 + 1, 2 ** 32 + 12345):
        bx, by = O.partition64(rp, 1, 0, dd, dd)
        xr = int(np.searchsorted(s, dd, side="right") - 1)
        assert (int(bx[0]), int(by[0])) == (xr, dd - xr)


# --------------------------------------------------------------------------------
# O6: Alg. 2
# --------------------------------------------------------------------------------
def split_set(rp, cx, cy):
    P = len(cx) - 1
    m = len(rp) - 1
    return sorted({int(cx[p]) for p in range(1, P) if cx[p] < m and cy[p] > rp[cx[p]]})


def test_o6_alg2_equals_o1_exact_and_counters():
    rs = np.random.RandomState(9)
    for trial in range(300):
        g = rand_graph(rs, rs.randint(0, 60), 30, 9, dup=bool(trial % 3 == 0), seed=trial)
        B = G.dense_int(30, int(rs.randint(1, 4)), seed=trial)
        M = g.m + g.nnz
        P = int(rs.randint(1, 30))
        L = max(1, -(-M // P)) if M else 0
        cx, cy = O.partition(g.row_ptr, P, L)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        C, na, nr = O.alg2_emulate(g.row_ptr, g.col_idx, g.val, B, cx, cy)
        assert np.array_equal(C, ref)
        S = split_set(g.row_ptr, cx, cy)
        inside = sum(1 for p in range(1, P) if cx[p] < g.m and cy[p] > g.row_ptr[cx[p]])
        assert nr == g.m - len(S)                 # every other row stored once (line 15)
        assert na == inside + len(S)              # a row cut k times is k+1 pieces
        # garbage prefill: exactly the split rows come out wrong (need zero-init)
        Cn, _, _ = O.alg2_emulate(g.row_ptr, g.col_idx, g.val, B, cx, cy,
                                  C_init=np.full((g.m, B.shape[1]), np.nan))
        bad = sorted(np.nonzero(np.isnan(Cn).any(axis=1))[0].tolist())
        assert bad == S


def test_o6_fig3_thread2_writes():
    rp = np.array([0, 8, 12, 13, 14, 15, 15, 16, 16, 16, 16], np.int32)
    g = G.random_csr(10, 10, np.diff(rp).astype(np.int32), 1)
    assert np.array_equal(g.row_ptr, rp)
    cx, cy = O.partition(rp, 4, 7)
    B = G.dense_int(10, 2, seed=1)
    # thread 2 alone: one atomic for its partial start row, one regular store (row 1)
    C, na, nr = O.alg2_emulate(rp, g.col_idx, g.val, B, cx[1:3], cy[1:3],
                               C_init=np.zeros((10, 2)))
    assert (na, nr) == (1, 1)


# --------------------------------------------------------------------------------
# O7: sharding (north-star stage 4)
# --------------------------------------------------------------------------------
def test_o7_shard_assembly_exact():
    rs = np.random.RandomState(10)
    for trial in range(150):
        g = rand_graph(rs, rs.randint(0, 50), 40, 10, seed=trial)
        B = G.dense_int(40, 3, seed=trial)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        world = int(rs.choice([1, 2, 3, 4, 8]))
        X, Y, T = O.shard(g.row_ptr, world)
        M = g.m + g.nnz
        per = -(-M // world)
        cx, cy = O.partition(g.row_ptr, world, per)
        assert np.array_equal(X, cx) and np.array_equal(Y, cy)
        out = np.zeros_like(ref)
        tails = []
        for r in range(world):
            Cl, tail = O.shard_local(g.row_ptr, g.col_idx, g.val, B, X, Y, r)
            out[X[r]:X[r + 1]] = Cl
            tails.append(tail)
            if T[r] >= 0:
                assert T[r] == X[r + 1] and Y[r + 1] > g.row_ptr[X[r + 1]]
            else:
                assert not np.any(tail)
        for h in range(world):            # owner(r) = max{g : X_g <= r}, ascending h
            if T[h] >= 0:
                owner = max(gg for gg in range(world) if X[gg] <= T[h])
                assert X[owner] <= T[h] < (X[owner + 1] if owner + 1 <= world else g.m) or \
                    X[owner] == T[h]
                out[T[h]] += tails[h]
        assert np.array_equal(out, ref)


def test_o7_owner_consumes_row_end():
    rs = np.random.RandomState(11)
    for trial in range(100):
        g = rand_graph(rs, rs.randint(1, 40), 40, 8, seed=trial)
        xs, ys = O.merge_walk(g.row_ptr)
        world = int(rs.choice([2, 4, 8]))
        X, Y, _ = O.shard(g.row_ptr, world)
        D = X.astype(np.int64) + Y
        for r in range(g.m):
            # the merge item that consumes row end r is the step where x goes r -> r+1
            step = int(np.nonzero(xs == r + 1)[0][0])        # coordinate after the item
            shard = int(np.searchsorted(D, step, side="left")) - 1  # D_g < step <= D_{g+1}
            owner = max(gg for gg in range(world) if X[gg] <= r)
            assert shard == owner


def test_o4_plan_thread_floor_p139():
    """"When the computed threads are below a threshold (e.g., 1024), the total
    thread count is set to the threshold value" -- "the merge path cost is decreased to
    ensure a minimum number of threads".  Checked by brute force: with the threshold in
    force the thread count equals it and the items per thread are the SMALLEST count
    that lets 1024 threads cover the merge path (found by search, not by formula), never
    above the requested cost; above the threshold the cost is kept.  The partition of a
    random CSR of that size then covers the merge path with segments of <= L items."""
    rs = np.random.RandomState(139)
    for M_items, cost in [(10_000, 20), (1_500, 50), (1023, 1), (13_264, 64), (100_000, 64)]:
        m = M_items // 3
        nnz = M_items - m
        P, L = O.plan(m, nnz, cost, 1024)
        threads_from_cost = -(-M_items // cost)           # merge_items / cost
        if threads_from_cost < 1024:
            assert P == 1024
            assert L == min(l for l in range(1, cost + 1) if 1024 * l >= M_items)
            assert L <= cost                                # the cost is decreased
        else:
            assert P == threads_from_cost and L <= cost
        rl = rs.multinomial(nnz, np.ones(m) / m).astype(np.int32)
        rp = np.concatenate([[0], np.cumsum(rl)]).astype(np.int32)
        cx, cy = O.partition(rp, P, L)
        d = cx.astype(np.int64) + cy
        assert d[0] == 0 and d[-1] == M_items and np.all(np.diff(d) >= 0)
        assert np.all(np.diff(d) <= L)


def test_o9_xw_pins():
    """O9 (combination X*W and the ReLU of sigma(A X W)) pinned by: identity W;
    one-hot rows of X selecting rows of W (catches a transposed W); all-ones X giving the
    column sums of W (np.sum); a pure-Python triple loop on a tiny case; ReLU as the
    elementwise max with 0 of that brute force; rank-1 X = u v^T giving u (v^T W)."""
    rs = np.random.RandomState(9)
    X = rs.randn(7, 5).astype(np.float32)
    assert np.array_equal(O.xw_f64(X, np.eye(5, dtype=np.float32)), X.astype(np.float64))
    W = rs.randn(5, 3).astype(np.float32)
    E = np.eye(5, dtype=np.float32)[[4, 0, 2]]
    assert np.array_equal(O.xw_f64(E, W), W[[4, 0, 2]].astype(np.float64))
    Wi = rs.randint(-5, 6, size=(9, 4)).astype(np.float32)
    assert np.array_equal(O.xw_f64(np.ones((3, 9), np.float32), Wi),
                          np.tile(Wi.astype(np.float64).sum(0), (3, 1)))
    Xs = rs.randint(-3, 4, size=(4, 6)).astype(np.float32)
    Ws = rs.randint(-3, 4, size=(6, 5)).astype(np.float32)
    bf = np.array([[sum(float(Xs[i, f]) * float(Ws[f, j]) for f in range(6)) for j in range(5)]
                   for i in range(4)])
    assert np.array_equal(O.xw_f64(Xs, Ws), bf)
    assert np.array_equal(O.xw_f64(Xs, Ws, relu=True), np.where(bf > 0, bf, 0.0))
    u = rs.randint(-2, 3, size=8).astype(np.float32)
    v = rs.randint(-2, 3, size=6).astype(np.float32)
    vW = [sum(float(v[f]) * float(Ws[f, j]) for f in range(6)) for j in range(5)]
    assert np.array_equal(O.xw_f64(np.outer(u, v).astype(np.float32), Ws),
                          np.array([[float(ui) * x for x in vW] for ui in u]))
