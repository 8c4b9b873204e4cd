"""GPU parity of the NEXT-4 64-bit-index path (mps_csr64: int64 row_ptr and nnz
coordinates) against the CPU oracle, through the C ABI.

Bars as for the int32 path: coordinates bit-exact against
oracle O4 (oracle_partition64); integer-valued inputs bit-exact against O1 in every
fix-up mode; float inputs within |C - C_ref| <= 1e-5 (|A||B|) + 1e-7.  The large cases
go past 2^31 non-zeros and compare sampled rows (recomputed on the host from the same
counter-based generator) plus properties that hold at any size.
"""
import numpy as np
import pytest
import torch

import graphgen as G
import oracle as O

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_ispass_shangndk23_b200 as M
    from paper_conf_ispass_shangndk23_b200 import api


def dev64(g):
    t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).cuda()
    return M.CSR(t(g.row_ptr.astype(np.int64)), t(g.col_idx), t(g.val), g.n)


def rand_graph(rs, m, n, max_len, seed, dup=False, vals="int"):
    rl = rs.randint(0, max_len + 1, size=m)
    if m and rs.rand() < 0.5:
        rl[rs.randint(m)] = max_len * 30       # an evil row
    if m and rs.rand() < 0.5:
        rl[rs.rand(m) < 0.4] = 0               # empty rows
    return G.random_csr(m, n, rl.astype(np.int32), seed, canonical=not dup, values=vals)


def test_partition64_bit_exact_small():
    rs = np.random.RandomState(0)
    for trial in range(40):
        g = rand_graph(rs, int(rs.randint(0, 400)), 60, 10, seed=trial)
        A = dev64(g)
        M_ = g.m + g.nnz
        b = int(rs.randint(0, M_ + 1))
        e = int(rs.randint(b, M_ + 1))
        P = int(rs.randint(1, 80))
        L = int(rs.randint(0, 2 * max(1, (e - b) // P) + 2))
        cx, cy = M.partition(A, P, L, b, e)
        assert cy.dtype == torch.int64
        ox, oy = O.partition64(g.row_ptr.astype(np.int64), P, L, b, e)
        assert np.array_equal(cx.cpu().numpy(), ox) and np.array_equal(cy.cpu().numpy(), oy)


def test_partition64_beyond_2p31_bit_exact():
    """Only row_ptr is needed: m = 1M rows, nnz ~ 5e9 (> 2^32), bit-exact vs O4-64."""
    rs = np.random.RandomState(1)
    m = 1_000_000
    rl = rs.randint(0, 9000, size=m).astype(np.int64)
    rl[rs.randint(m, size=3)] = 700_000_000           # rows that alone cross 2^31 offsets
    rp = np.zeros(m + 1, np.int64)
    np.cumsum(rl, out=rp[1:])
    nnz = int(rp[-1])
    assert m + nnz > 2 ** 32
    rpd = torch.from_numpy(rp).cuda()
    cx = torch.empty(0)
    for cost in (256, 2048, 1 << 20):
        P, L = M.plan(m, nnz, 64, 0, cost, 1, wide=True)
        assert (P, L) == O.plan(m, nnz, cost, 1)
        cx = torch.empty(P + 1, dtype=torch.int32, device="cuda")
        cy = torch.empty(P + 1, dtype=torch.int64, device="cuda")
        M.mps_partition64(api._p(rpd), m, nnz, 0, m + nnz, P, L, api._p(cx), api._p(cy),
                          api._stream())
        ox, oy = O.partition64(rp, P, L)
        assert np.array_equal(cx.cpu().numpy(), ox) and np.array_equal(cy.cpu().numpy(), oy)


@pytest.mark.parametrize("fixup", ["atomic", "carry"])
@pytest.mark.parametrize("K", [1, 4, 16, 17, 64, 128, 256, 520])
def test_spmm64_integer_exact(fixup, K):
    rs = np.random.RandomState(K)
    for trial in range(3):
        g = rand_graph(rs, int(rs.randint(1, 500)), 300, 12, seed=trial, dup=bool(trial % 2))
        B = G.dense_int(300, K, seed=trial)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        A = dev64(g)
        Bt = torch.from_numpy(B).cuda()
        for cost in (1, 7, 256, 10 ** 6):
            sch = M.Schedule.build(A, K, items_per_part=cost, min_parts=1)
            assert sch.coord_y.dtype == torch.int64
            C = torch.full((g.m, K), float("nan"), device="cuda")
            M.spmm(A, Bt, schedule=sch, fixup=fixup, out=C)
            assert np.array_equal(C.cpu().numpy().astype(np.float64), ref), (trial, cost)
            C2 = M.spmm(A, Bt, fixup=fixup, items_per_part=cost, min_parts=1)
            assert np.array_equal(C2.cpu().numpy().astype(np.float64), ref), (trial, cost)
            C3 = M.spmm(A, Bt.to(torch.bfloat16), fixup=fixup, items_per_part=cost, min_parts=1)
            assert np.array_equal(C3.cpu().numpy().astype(np.float64), ref), (trial, cost)


@pytest.mark.parametrize("fixup", ["atomic", "carry"])
def test_spmm64_float_tolerance_relu_and_stats(fixup):
    g = G.workload("pubmed")
    K = 64
    B = G.features("pubmed", K)
    ref, bnd = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B)
    A = dev64(g)
    C = M.spmm(A, torch.from_numpy(B).cuda(), fixup=fixup)
    r = O.check(C.cpu().numpy(), ref, bnd)
    assert r["ok"], r
    Cr = M.spmm(A, torch.from_numpy(B).cuda(), fixup=fixup, epilogue="relu")
    r = O.check(Cr.cpu().numpy(), np.maximum(ref, 0), bnd)
    assert r["ok"], r
    # Fig. 5 statistic equals the int32 path's and the oracle's counters (O6)
    sch = M.Schedule.build(A, K, items_per_part=97, min_parts=1)
    a64 = M.write_stats(A, sch)
    A32 = M.CSR.from_numpy(g.row_ptr, g.col_idx, g.val, g.n)
    s32 = M.Schedule.build(A32, K, items_per_part=97, min_parts=1)
    assert a64 == M.write_stats(A32, s32)
    ox, oy = O.partition(g.row_ptr, sch.num_parts, sch.items_per_part)
    _, na, nr = O.alg2_emulate(g.row_ptr, g.col_idx, g.val, B[:, :1], ox, oy)
    assert a64 == (na, nr)


def test_validate_csr64():
    g = rand_graph(np.random.RandomState(3), 50, 40, 6, seed=3)
    A = dev64(g)
    assert M.validate_csr(A) == -1
    A.col_idx[5] = 40
    assert M.validate_csr(A) == g.m + 1 + 5


def test_int32_entry_points_reject_wide_sizes():
    P, L = M.plan(10, 2 ** 31, 16, 0, 0, 0, wide=True)
    assert P * L >= 10 + 2 ** 31
    with pytest.raises(M.MpsError):
        M.plan(10, 2 ** 31, 16)


# --------------------------------------------------------------------------------
# nnz > 2^31 end to end: sampled rows against O1 (bit-exact, integer inputs) and the
# partition's unique-point property at full size.
# --------------------------------------------------------------------------------
def wide_case(K, seed=41):
    m, n = 2_621_440, 1 << 20
    evil = [(0, 1_000_000), (m // 2 + 3, 1_000_000), (m - 1, 1_000_000)]
    rp = G.wide_row_ptr(m, 2048, seed, evil)
    # one more long row straddling non-zero 2^31
    r31 = int(np.searchsorted(rp, 2 ** 31, side="right") - 1)
    return m, n, rp, r31


@pytest.mark.parametrize("b_dtype", ["f32", "bf16"])
def test_spmm64_beyond_2p31_sampled_rows(b_dtype):
    K, seed = 16, 41
    m, n, rp, r31 = wide_case(K, seed)
    nnz = int(rp[-1])
    assert nnz > 2 ** 31 + 2 ** 29
    col, val = G.wide_cols_vals_device(nnz, n, seed)
    Bh = G.dense_int(n, K, seed=seed)
    Bt = torch.from_numpy(Bh).cuda()
    if b_dtype == "bf16":
        Bt = Bt.to(torch.bfloat16)
    A = M.CSR(torch.from_numpy(rp).cuda(), col, val, n)
    for fixup in ("atomic", "carry"):
        sch = M.Schedule.build(A, K, b_dtype=Bt.dtype)
        # unique-point property of every coordinate (readings R4/R5), on the device
        rpd = A.row_ptr
        x = sch.coord_x.long()
        y = sch.coord_y
        assert torch.all(rpd[x] <= y)
        inner = x < m
        assert torch.all(y[inner] <= rpd[x[inner] + 1])
        d = torch.clamp(torch.arange(sch.num_parts + 1, device="cuda") * sch.items_per_part,
                        max=m + nnz)
        assert torch.equal(x + y, d)
        C = torch.full((m, K), float("nan"), device="cuda")
        M.spmm(A, Bt, schedule=sch, fixup=fixup, out=C)
        torch.cuda.synchronize()
        assert not torch.isnan(C).any()
        rs = np.random.RandomState(7)
        rows = np.unique(np.concatenate([
            rs.randint(0, m, size=300), [0, 1, m // 2 + 3, m - 2, m - 1, r31 - 1, r31, r31 + 1],
            # rows cut by segment boundaries near 2^31
            sch.coord_x.cpu().numpy()[np.searchsorted(sch.coord_y.cpu().numpy(), 2 ** 31) - 2:][:6]
            .clip(0, m - 1)]))
        lens = rp[rows + 1] - rp[rows]
        js = np.concatenate([np.arange(rp[r], rp[r + 1]) for r in rows])
        ci, cv = G.wide_cols_vals_host(js, n, seed)
        mini_rp = np.zeros(len(rows) + 1, np.int64)
        np.cumsum(lens, out=mini_rp[1:])
        ref = O.csr_spmm_f64(mini_rp.astype(np.int32), ci, cv, Bh, want_bound=False)
        got = C[torch.from_numpy(rows).cuda()].cpu().numpy().astype(np.float64)
        assert np.array_equal(got, ref), (fixup, b_dtype)
        del C
    torch.cuda.empty_cache()
