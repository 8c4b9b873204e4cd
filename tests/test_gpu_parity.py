"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bars: merge-path coordinates bit-exact; integer-valued inputs
bit-exact in every fix-up mode, schedule and shard count; float inputs within the
north-star tolerance |C - C_ref| <= 1e-5 (|A||B|) + 1e-7 (oracle.check, O8).
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


def dev(g):
    return M.CSR.from_numpy(g.row_ptr, g.col_idx, g.val, g.n)


def tB(B, dtype=torch.float32):
    return torch.from_numpy(B).to("cuda").to(dtype)


def rand_graph(rs, m, n, max_len, seed, dup=False, vals="int"):
    kind = rs.randint(4)
    if kind == 0:
        rl = rs.randint(0, max_len + 1, size=m)
    elif kind == 1:
        rl = np.where(rs.rand(m) < 0.6, 0, rs.randint(0, max_len + 1, size=m))
    elif kind == 2:
        rl = rs.randint(0, 3, size=m)
        if m:
            rl[rs.randint(m)] = max_len * 20
    else:
        rl = rs.randint(0, max_len + 1, size=m)
        if m:
            rl[0] = max_len * 10
            rl[-1] = max_len * 10
    return G.random_csr(m, n, rl.astype(np.int32), seed, canonical=not dup, values=vals)


# --------------------------------------------------------------------------------
# a2: partition, bit-exact
# --------------------------------------------------------------------------------
@pytest.mark.parametrize("name", ["cora", "pubmed"])
@pytest.mark.parametrize("cost", [1, 7, 64, 512, 100000])
def test_partition_bit_exact_workloads(name, cost):
    g = G.workload(name)
    A = dev(g)
    P, L = M.plan(g.m, g.nnz, 16, 0, cost, 1)
    assert (P, L) == O.plan(g.m, g.nnz, cost, 1)
    cx, cy = M.partition(A, P, L)
    ox, oy = O.partition(g.row_ptr, P, L)
    assert np.array_equal(cx.cpu().numpy(), ox) and np.array_equal(cy.cpu().numpy(), oy)


def test_partition_bit_exact_random_and_subranges():
    rs = np.random.RandomState(0)
    for trial in range(60):
        g = rand_graph(rs, int(rs.randint(0, 300)), 50, 9, seed=trial)
        A = dev(g)
        M_ = g.m + g.nnz
        b = int(rs.randint(0, M_ + 1))
        e = int(rs.randint(b, M_ + 1))
        P = int(rs.randint(1, 70))
        L = int(rs.randint(0, 2 * max(1, (e - b) // P) + 2))
        cx, cy = M.partition(A, P, L, b, e)
        ox, oy = O.partition(g.row_ptr, P, L, b, e)
        assert np.array_equal(cx.cpu().numpy(), ox) and np.array_equal(cy.cpu().numpy(), oy)


def test_partition_split_zeroes_exactly_cut_rows():
    rs = np.random.RandomState(4)
    for trial in range(20):
        g = rand_graph(rs, int(rs.randint(1, 300)), 40, 9, seed=trial)
        A = dev(g)
        P = int(rs.randint(1, 60))
        L = -(-(g.m + g.nnz) // P)
        K = 7
        C = torch.full((g.m, K + 3), float("nan"), device="cuda")
        cx = torch.empty(P + 1, dtype=torch.int32, device="cuda")
        cy = torch.empty_like(cx)
        M.mps_partition_split(api._p(A.row_ptr), g.m, g.nnz, P, L, api._p(cx), api._p(cy),
                              api._p(C), K + 3, K, api._stream())
        ox, oy = O.partition(g.row_ptr, P, L)
        assert np.array_equal(cx.cpu().numpy(), ox) and np.array_equal(cy.cpu().numpy(), oy)
        cut = sorted({int(ox[p]) for p in range(P + 1) if ox[p] < g.m and oy[p] > g.row_ptr[ox[p]]})
        Ch = C.cpu().numpy()
        zeroed = sorted(np.nonzero(~np.isnan(Ch[:, :K]).any(axis=1))[0].tolist())
        assert zeroed == cut
        assert np.all(Ch[cut, :K] == 0) and np.isnan(Ch[:, K:]).all()


def test_partition_fig3():
    rp = np.array([0, 8, 12, 13, 14, 15, 15, 16, 16, 16, 16], np.int32)
    g = G.random_csr(10, 10, np.diff(rp).astype(np.int32), 1)
    cx, cy = M.partition(dev(g), 4, 7)
    assert cx.cpu().tolist() == [0, 0, 2, 6, 10] and cy.cpu().tolist()[:3] == [0, 7, 12]


# --------------------------------------------------------------------------------
# a3 + a4: SpMM, integer inputs bit-exact
# --------------------------------------------------------------------------------
KS = [1, 3, 4, 15, 16, 17, 32, 64, 100, 128, 256, 257, 520]


@pytest.mark.parametrize("fixup", ["atomic", "carry"])
@pytest.mark.parametrize("K", KS)
def test_spmm_integer_exact_random(fixup, K):
    rs = np.random.RandomState(K)
    for trial in range(6):
        g = rand_graph(rs, int(rs.randint(1, 400)), 300, 12, seed=trial, dup=bool(trial % 2))
        B = G.dense_int(300, K, seed=trial)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        A = dev(g)
        for cost in (1, 5, 33, 256, 10 ** 6):
            sch = M.Schedule.build(A, K, items_per_part=cost, min_parts=1)
            C = torch.full((g.m, K), float("nan"), device="cuda")
            M.spmm(A, tB(B), schedule=sch, fixup=fixup, out=C)
            assert np.array_equal(C.cpu().numpy().astype(np.float64), ref), (trial, cost)
            C2 = M.spmm(A, tB(B), fixup=fixup, items_per_part=cost, min_parts=1)
            assert np.array_equal(C2.cpu().numpy().astype(np.float64), ref), (trial, cost)


@pytest.mark.parametrize("fixup", ["atomic", "carry"])
@pytest.mark.parametrize("K", [1, 2, 8, 16, 24, 32, 64, 128, 256, 264, 1032])
def test_spmm_bf16_integer_exact(fixup, K):
    """B in {-4..4} is exact in bf16, so the bf16-B path (a5) must match O1 bit-exactly."""
    rs = np.random.RandomState(100 + K)
    for trial in range(3):
        g = rand_graph(rs, int(rs.randint(1, 500)), 200, 12, seed=trial, dup=bool(trial % 2))
        B = G.dense_int(200, K, seed=trial)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        A = dev(g)
        for cost in (1, 13, 300, 10 ** 6):
            C = torch.full((g.m, K), float("nan"), device="cuda")
            M.spmm(A, tB(B, torch.bfloat16), fixup=fixup, out=C, items_per_part=cost, min_parts=1)
            assert np.array_equal(C.cpu().numpy().astype(np.float64), ref), (trial, cost)


@pytest.mark.parametrize("fixup", ["atomic", "carry"])
def test_spmm_padded_and_misaligned(fixup):
    rs = np.random.RandomState(3)
    g = rand_graph(rs, 500, 200, 10, seed=3)
    A = dev(g)
    for K, ld, off in [(64, 72, 0), (64, 68, 1), (30, 33, 0), (128, 130, 2), (16, 20, 3)]:
        Bfull = G.dense_int(200, ld, seed=K)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, np.ascontiguousarray(Bfull[:, off:off + K]),
                             want_bound=False)
        Bt = tB(Bfull)[:, off:off + K]          # row stride ld, base offset by `off` floats
        Cbig = torch.full((g.m, K + 5), float("nan"), device="cuda")
        C = Cbig[:, 1:1 + K]                    # ldc = K + 5, misaligned base
        M.spmm(A, Bt, fixup=fixup, out=C, items_per_part=37, min_parts=1)
        assert np.array_equal(C.cpu().numpy().astype(np.float64), ref), (K, ld, off)
        assert torch.isnan(Cbig[:, 0]).all() and torch.isnan(Cbig[:, K + 1:]).all()


@pytest.mark.parametrize("fixup", ["atomic", "carry"])
def test_spmm_degenerate(fixup):
    K = 8
    cases = []
    cases.append(G.random_csr(0, 5, np.zeros(0, np.int32), 1))            # m = 0
    cases.append(G.random_csr(7, 5, np.zeros(7, np.int32), 1))            # nnz = 0
    for pos in (0, 3, 6):                                                 # one row holds all
        rl = np.zeros(7, np.int32)
        rl[pos] = 3000
        cases.append(G.random_csr(7, 50, rl, pos))
    for L in (9, 10, 11):                                                 # rows L-1, L, L+1
        rl = np.full(40, L - 1, np.int32)
        cases.append(G.random_csr(40, 50, rl, L))
    for g in cases:
        B = G.dense_int(g.n, K, seed=2)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        A = dev(g)
        for cost, pmin in [(1, 1), (10, 1), (10 ** 6, 1), (4, 10 ** 4)]:   # L = 1, P > M
            C = torch.full((g.m, K), float("nan"), device="cuda")
            M.spmm(A, tB(B), fixup=fixup, out=C, items_per_part=cost, min_parts=pmin)
            assert np.array_equal(C.cpu().numpy().astype(np.float64), ref)


def test_identity_and_ones():
    n, K = 3001, 64
    rp = np.arange(n + 1, dtype=np.int32)
    A = M.CSR.from_numpy(rp, np.arange(n, dtype=np.int32), np.ones(n, np.float32), n)
    B = G.dense_uniform(n, K, seed=5)
    C = M.spmm(A, tB(B))
    assert torch.equal(C.cpu(), torch.from_numpy(B))
    g = G.workload("pubmed")
    C1 = M.spmm(dev(g), torch.ones(g.n, 16, device="cuda")).cpu().numpy()
    rows = np.repeat(np.arange(g.m), np.diff(g.row_ptr))
    wdeg = np.bincount(rows, weights=g.val.astype(np.float64), minlength=g.m)
    assert np.all(C1 == C1[:, :1])
    np.testing.assert_allclose(C1[:, 0], wdeg, rtol=1e-5, atol=1e-7)


# --------------------------------------------------------------------------------
# float inputs within the north-star tolerance
# --------------------------------------------------------------------------------
@pytest.mark.parametrize("name,K", [("cora", 16), ("pubmed", 16), ("pubmed", 64)])
@pytest.mark.parametrize("fixup", ["atomic", "carry"])
def test_spmm_tolerance_workloads(name, K, fixup):
    g = G.workload(name)
    B = G.features(name, K)
    ref, bnd = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B)
    A = dev(g)
    for cost in (0, 8, 64):
        C = torch.full((g.m, K), float("nan"), device="cuda")
        M.spmm(A, tB(B), fixup=fixup, out=C, items_per_part=cost)
        r = O.check(C.cpu().numpy(), ref, bnd)
        assert r["ok"], r


def test_captured_graph_replay():
    g = G.workload("cora")
    B = G.features("cora", 16)
    ref, bnd = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B)
    A = dev(g)
    Bd = tB(B)
    cap = M.CapturedSpMM(A, Bd)
    for _ in range(3):
        cap.C.fill_(float("nan"))
        C = cap()
        torch.cuda.synchronize()
        assert O.check(C.cpu().numpy(), ref, bnd)["ok"]
    Bd.mul_(2.0)                               # new B values, same buffer
    C = cap()
    torch.cuda.synchronize()
    assert O.check(C.cpu().numpy(), 2 * ref, 2 * bnd)["ok"]


def _hot_bitmap(A, budget):
    import ctypes
    nb = ctypes.c_size_t()
    M.mps_hot_rows_workspace_bytes(A.n, ctypes.byref(nb))
    ws = torch.empty(max(nb.value, 1), dtype=torch.uint8, device="cuda")
    bm = torch.zeros((A.n + 31) // 32, dtype=torch.int32, device="cuda")
    a = A.struct()
    M.mps_hot_rows(ctypes.byref(a), budget, api._p(bm), api._p(ws), nb.value, api._stream())
    return bm


def test_hot_rows_bitmap_rule():
    g = G.workload("pubmed")
    A = dev(g)
    counts = np.bincount(g.col_idx, minlength=g.n)
    for budget in (0, 10, 500, 5000, 10 ** 6):
        bm = _hot_bitmap(A, budget).cpu().numpy().view(np.uint32)
        hot = ((bm[np.arange(g.n) >> 5] >> (np.arange(g.n) & 31)) & 1).astype(bool)
        # reference rule: smallest power of two t with #{count >= t} <= budget
        thr = None
        for b in range(32, 0, -1):
            t = 1 << (b - 1)
            if np.count_nonzero(counts >= t) > budget:
                break
            thr = t
        ref = counts >= thr if thr is not None else np.zeros(g.n, bool)
        assert np.array_equal(hot, ref), budget
        assert hot.sum() <= budget


@pytest.mark.parametrize("fixup", ["atomic", "carry"])
def test_spmm_segments_hot_exact(fixup):
    import ctypes
    rs = np.random.RandomState(21)
    for K in (8, 64, 128, 200):
        g = rand_graph(rs, 700, 300, 12, seed=K)
        B = G.dense_int(300, K, seed=K)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        A = dev(g)
        sch = M.Schedule.build(A, K, items_per_part=50, min_parts=1)
        bm = _hot_bitmap(A, 40)
        C = torch.full((g.m, K), float("nan"), device="cuda")
        a = A.struct()
        Bt = tB(B)
        nb = ctypes.c_size_t()
        M.mps_spmm_workspace_bytes(ctypes.byref(a), K, 0, sch.num_parts, api._fix(fixup),
                                   ctypes.byref(nb))
        ws = torch.empty(max(nb.value, 1), dtype=torch.uint8, device="cuda")
        if fixup == "atomic":
            M.mps_zero_split_rows(ctypes.byref(a), api._p(sch.coord_x), api._p(sch.coord_y),
                                  sch.num_parts, api._p(C), K, K, api._stream())
        M.mps_spmm_segments_hot(ctypes.byref(a), api._p(Bt), 0, K, K, api._p(C), K,
                                api._p(sch.coord_x), api._p(sch.coord_y), sch.num_parts,
                                api._fix(fixup), api._p(bm), api._p(ws), nb.value, api._stream())
        assert np.array_equal(C.cpu().numpy().astype(np.float64), ref), K


def test_online_hot_path_large_B(monkeypatch):
    """With MPS_HOT_FRAC set, B larger than half the L2 switches the online path to
    hot-row residency (the env is read once per process: run this in a subprocess)."""
    import subprocess, sys, os
    code = "import sys; sys.path.insert(0, %r); import tests.test_gpu_parity as t; t._online_hot_body()" % \
        os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, MPS_HOT_FRAC="0.6")
    r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True)
    assert r.returncode == 0, r.stdout + r.stderr


def _online_hot_body():
    import ctypes
    n, K = 300000, 256                          # 307 MB of fp32 B
    rl = np.random.RandomState(3).randint(0, 8, size=n).astype(np.int32)
    g = G.random_csr(n, n, rl, 5)
    A = dev(g)
    hot = ctypes.c_int64()
    a = A.struct()
    M.mps_hot_budget_rows(ctypes.byref(a), K, 0, ctypes.byref(hot))
    assert hot.value > 0
    B = G.dense_int(n, K, seed=2)
    C = M.spmm(A, tB(B))
    rows = np.random.RandomState(1).choice(n, 2000, replace=False)
    ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, rows=rows, want_bound=False)
    assert np.array_equal(C[torch.from_numpy(rows).cuda()].cpu().numpy().astype(np.float64), ref)


@pytest.mark.parametrize("fixup", ["atomic", "carry"])
def test_relu_epilogue_exact(fixup):
    """MPS_EPI_RELU == max(A*B, 0) bit-exactly on integer inputs, for complete and cut rows,
    offline and online, fp32 and bf16 B."""
    rs = np.random.RandomState(31)
    for K in (8, 64, 96, 256):
        g = rand_graph(rs, 600, 200, 14, seed=K)
        B = G.dense_int(200, K, seed=K)
        ref = np.maximum(O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False), 0)
        A = dev(g)
        for dt in (torch.float32, torch.bfloat16):
            for cost in (5, 60):
                sch = M.Schedule.build(A, K, dt, items_per_part=cost, min_parts=1)
                C = torch.full((g.m, K), float("nan"), device="cuda")
                M.spmm(A, tB(B, dt), schedule=sch, fixup=fixup, out=C, epilogue="relu")
                assert np.array_equal(C.cpu().numpy().astype(np.float64), ref), (K, dt, cost)
                C2 = M.spmm(A, tB(B, dt), fixup=fixup, items_per_part=cost, min_parts=1,
                            epilogue="relu")
                assert np.array_equal(C2.cpu().numpy().astype(np.float64), ref), (K, dt, cost)


@pytest.mark.parametrize("online", [False, True])
def test_gcn2_layers_against_oracle(online):
    """2-layer GCN (NEXT-2): each aggregation checked against O1 on the GPU-computed X*W."""
    g = G.workload("pubmed")
    A = dev(g)
    gen = torch.Generator(device="cpu").manual_seed(0)
    X = torch.randn(g.n, 128, generator=gen).cuda()
    W1 = (torch.randn(128, 64, generator=gen) / 11).cuda()
    W2 = (torch.randn(64, 16, generator=gen) / 8).cuda()
    net = M.GCN2(A, W1, W2, online=online, combination="cublas")
    out = net(X)
    torch.cuda.synchronize()
    B1 = (X @ W1).cpu().numpy()
    ref1, bnd1 = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B1)
    H = net.H.cpu().numpy()
    r = O.check(H, np.maximum(ref1, 0), bnd1)
    assert r["ok"], r
    B2 = (net.H @ W2).cpu().numpy()
    ref2, bnd2 = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B2)
    r = O.check(out.cpu().numpy(), ref2, bnd2)
    assert r["ok"], r


def test_gcn2_tcgen05_combination():
    """NEXT-3: X*W on tcgen05 (bf16 B) feeding the SpMM; each stage checked."""
    g = G.workload("pubmed")
    A = dev(g)
    gen = torch.Generator(device="cpu").manual_seed(1)
    X = torch.randn(g.n, 128, generator=gen).cuda()
    W1 = (torch.randn(128, 64, generator=gen) / 11).cuda()
    W2 = (torch.randn(64, 16, generator=gen) / 8).cuda()
    net = M.GCN2(A, W1, W2)                  # combination="auto" -> tcgen05 here
    assert net.combination == "tcgen05"
    out = net(X)
    torch.cuda.synchronize()
    # layer 1: B1 = bf16(X) * bf16(W1) in fp32, rounded to bf16, checked vs fp64
    Xb, W1b = X.to(torch.bfloat16).double().cpu(), W1.to(torch.bfloat16).double().cpu()
    B1 = M.xw_bf16(X.to(torch.bfloat16), net.W1t)
    ref = torch.from_numpy(O.xw_f64(Xb.numpy(), W1b.numpy()))            # O9
    bnd = torch.from_numpy(O.xw_f64(Xb.abs().numpy(), W1b.abs().numpy()))
    assert torch.all((B1.double().cpu() - ref).abs() <= 2 ** -8 * ref.abs() + 1e-5 * bnd)
    # aggregation on exactly that bf16 B1, with the fused ReLU
    ref1, bnd1 = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B1.float().cpu().numpy())
    r = O.check(net.H.cpu().numpy(), np.maximum(ref1, 0), bnd1)
    assert r["ok"], r
    B2 = M.xw_bf16(net.H.to(torch.bfloat16), net.W2t)
    ref2, bnd2 = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B2.float().cpu().numpy())
    r = O.check(out.cpu().numpy(), ref2, bnd2)
    assert r["ok"], r


@pytest.mark.parametrize("fixup", ["atomic", "carry"])
def test_dynamic_segment_claims(monkeypatch, fixup):
    """More segments than resident warps: warps claim segments from a self-resetting
    grid counter (MPS_DYN=1, default) instead of the static stride (MPS_DYN=0).  Integer
    inputs bit-exact against the oracle for both, over repeated launches (the counter must
    come back to zero), empty-row runs, a CUDA-graph replay and the offline entry point."""
    rs = np.random.RandomState(17)
    rl = rs.randint(0, 9, size=30000).astype(np.int32)
    rl[rs.rand(30000) < 0.3] = 0                   # runs of empty rows -> empty segments
    rl[12345] = 20000                               # a row cut by many segments
    g = G.random_csr(30000, 5000, rl, 21)
    A = dev(g)
    for K, dt in ((64, torch.float32), (16, torch.float32), (32, torch.bfloat16)):
        B = G.dense_int(5000, K, seed=K)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        for dyn in ("1", "0"):
            monkeypatch.setenv("MPS_DYN", dyn)
            for cost in (2, 7):
                for _ in range(3):
                    C = M.spmm(A, tB(B, dt), fixup=fixup, items_per_part=cost, min_parts=1)
                    assert np.array_equal(C.cpu().numpy().astype(np.float64), ref), (K, dyn, cost)
                sch = M.Schedule.build(A, K, dt, items_per_part=cost, min_parts=1)
                C = M.spmm(A, tB(B, dt), schedule=sch, fixup=fixup)
                assert np.array_equal(C.cpu().numpy().astype(np.float64), ref), (K, dyn, cost)
    monkeypatch.setenv("MPS_DYN", "1")
    B = G.dense_int(5000, 64, seed=3)
    ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
    Bd = tB(B)
    cap = M.CapturedSpMM(A, Bd, fixup=fixup, items_per_part=3, min_parts=1)
    for _ in range(4):
        cap.C.fill_(float("nan"))
        C = cap()
        torch.cuda.synchronize()
        assert np.array_equal(C.cpu().numpy().astype(np.float64), ref)


@pytest.mark.parametrize("fixup", ["atomic", "carry"])
def test_deep_gather_variant(monkeypatch, fixup):
    """The deep-gather instantiation (2x gathers in flight, 2 CTAs/SM; chosen for fp32
    256-B row slices when B is DRAM-bound and rows are long) forced on with MPS_DEEP=1:
    integer inputs bit-exact, untiled K=64 and K=128/192 in 64-column tiles, static and
    dynamic segment claims."""
    monkeypatch.setenv("MPS_DEEP", "1")
    monkeypatch.setenv("MPS_TILE", "64")
    rs = np.random.RandomState(23)
    rl = rs.randint(0, 80, size=4000).astype(np.int32)
    rl[rs.rand(4000) < 0.2] = 0
    rl[100] = 3000
    g = G.random_csr(4000, 3500, rl, 31)
    A = dev(g)
    for K in (64, 128, 192):
        B = G.dense_int(3500, K, seed=K)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        for dyn in ("1", "0"):
            monkeypatch.setenv("MPS_DYN", dyn)
            for cost in (3, 64, 0):
                C = M.spmm(A, tB(B), fixup=fixup, items_per_part=cost, min_parts=1 if cost else 0)
                assert np.array_equal(C.cpu().numpy().astype(np.float64), ref), (K, dyn, cost)


@pytest.mark.parametrize("fixup", ["atomic", "carry"])
def test_bf16_next_batch_prefetch(monkeypatch, fixup):
    """The bf16 dynamic kernels' next-batch L2 prefetch (on by rule where the tile's B
    slice exceeds half the L2) forced on for a small graph with MPS_PF=1: it only moves
    data into L2, so integer inputs stay bit-exact against the oracle for K = 64 (four
    rows per instruction), 128 (two) and 256 (one 256-B slice per tile), batches that end
    at chunk and segment edges, empty-row runs and a long row."""
    monkeypatch.setenv("MPS_PF", "1")
    monkeypatch.setenv("MPS_DYN", "1")
    rs = np.random.RandomState(29)
    rl = rs.randint(0, 12, size=20000).astype(np.int32)
    rl[rs.rand(20000) < 0.4] = 0
    rl[777] = 9000
    g = G.random_csr(20000, 6000, rl, 37)
    A = dev(g)
    for K in (64, 128, 256):
        B = G.dense_int(6000, K, seed=K + 1)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        for cost in (5, 64, 0):
            C = M.spmm(A, tB(B, torch.bfloat16), fixup=fixup, items_per_part=cost,
                       min_parts=1 if cost else 0)
            assert np.array_equal(C.cpu().numpy().astype(np.float64), ref), (K, cost)


def test_carry_is_deterministic():
    g = G.workload("pubmed")
    B = tB(G.features("pubmed", 64))
    A = dev(g)
    a = M.spmm(A, B, fixup="carry", items_per_part=16)
    b = M.spmm(A, B, fixup="carry", items_per_part=16)
    assert torch.equal(a, b)


def test_bf16_B_within_tolerance():
    g = G.workload("pubmed")
    for K in (16, 64, 128, 256, 24):
        B = G.features("pubmed", K)
        Bb = torch.from_numpy(B).to(torch.bfloat16)
        Bq = Bb.to(torch.float32).numpy()              # the oracle sees the rounded B
        ref, bnd = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, Bq)
        for fixup in ("atomic", "carry"):
            C = M.spmm(dev(g), Bb.cuda(), fixup=fixup, items_per_part=50)
            r = O.check(C.cpu().numpy(), ref, bnd)
            assert r["ok"], (K, fixup, r)


# --------------------------------------------------------------------------------
# Fig. 5 statistic, validation, host end-to-end
# --------------------------------------------------------------------------------
def test_write_stats_match_alg2_counters():
    rs = np.random.RandomState(8)
    for trial in range(20):
        g = rand_graph(rs, int(rs.randint(1, 300)), 40, 9, seed=trial)
        A = dev(g)
        for cost in (1, 6, 50):
            sch = M.Schedule.build(A, 4, items_per_part=cost, min_parts=1)
            B = G.dense_int(40, 2, seed=1)
            _, na, nr = O.alg2_emulate(g.row_ptr, g.col_idx, g.val, B,
                                       sch.coord_x.cpu().numpy(), sch.coord_y.cpu().numpy())
            assert M.write_stats(A, sch) == (na, nr)


@pytest.mark.parametrize("fixup", ["atomic", "carry"])
@pytest.mark.parametrize("K", [4, 16, 64, 130, 256])
def test_kernel_write_counts_match_alg2(fixup, K):
    """NEXT-1, Fig. 5: the counters INSIDE the segment kernel (what it wrote)
    equal the oracle's serial Alg. 2 counters O6: issued + elided partial-row updates =
    #atomic, complete-row stores = #regular; C is bit-exact with integer inputs."""
    rs = np.random.RandomState(80 + K)
    for trial in range(10):
        g = rand_graph(rs, int(rs.randint(1, 500)), 60, 11, seed=trial)
        A = dev(g)
        B = G.dense_int(60, K, seed=trial)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        for cost in (1, 5, 23, 200):
            sch = M.Schedule.build(A, K, items_per_part=cost, min_parts=1)
            C, (issued, elided, regular) = M.write_counts(A, tB(B), sch, fixup=fixup)
            torch.cuda.synchronize()
            _, na, nr = O.alg2_emulate(g.row_ptr, g.col_idx, g.val, B[:, :1],
                                       sch.coord_x.cpu().numpy(), sch.coord_y.cpu().numpy())
            assert (issued + elided, regular) == (na, nr), (trial, cost)
            assert M.write_stats(A, sch) == (na, nr)
            assert np.array_equal(C.cpu().numpy().astype(np.float64), ref), (trial, cost)


def test_kernel_write_counts_full_size_reddit():
    """The statistic at full size on the bench's workload (Reddit K=64, default plan):
    kernel counters == O6 == mps_write_stats."""
    g = G.workload("reddit")
    A = dev(g)
    sch = M.Schedule.build(A, 64)
    B = torch.zeros((g.n, 64), device="cuda")
    _, (issued, elided, regular) = M.write_counts(A, B, sch)
    _, na, nr = O.alg2_emulate(g.row_ptr, g.col_idx, g.val, np.zeros((g.n, 1), np.float32),
                               sch.coord_x.cpu().numpy(), sch.coord_y.cpu().numpy())
    assert (issued + elided, regular) == (na, nr)
    cx, cy = sch.coord_x.cpu().numpy(), sch.coord_y.cpu().numpy()
    cut = np.unique(cx[(cx < g.m) & (cy > g.row_ptr[np.minimum(cx, g.m)])])
    assert regular == g.m - len(cut)         # every row not cut is stored exactly once


def test_validate_csr():
    g = G.workload("cora")
    assert M.validate_csr(dev(g)) == -1
    bad = g.col_idx.copy()
    bad[100] = g.n + 5
    assert M.validate_csr(M.CSR.from_numpy(g.row_ptr, bad, g.val, g.n)) == g.m + 1 + 100


def test_spmm_host_end_to_end():
    g = G.workload("pubmed")
    B = G.features("pubmed", 64)
    ref, bnd = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B)
    pin = lambda a: torch.from_numpy(a).pin_memory()
    C = M.spmm_host(pin(g.row_ptr), pin(g.col_idx), pin(g.val), g.n, pin(B))
    assert O.check(C.numpy(), ref, bnd)["ok"]


@pytest.mark.parametrize("chunk", [1, 4096, 65536, 0])
@pytest.mark.parametrize("case", ["pubmed", "evil", "empty_rows", "no_nnz"])
def test_spmm_host_pipelined_chunks(monkeypatch, chunk, case):
    """mps_spmm_host in atomic mode pipelines the H2D of A in merge-path chunks with the
    segment kernels and the D2H of finished rows (MPS_HOST_CHUNK_BYTES sets the chunk
    size; 1 byte = the 64-chunk cap).  Integer inputs: bit-exact against the oracle and
    against the serial path (MPS_HOST_SERIAL=1), for rows cut by every chunk boundary."""
    rs = np.random.RandomState(7)
    if case == "pubmed":
        g = G.workload("pubmed")
        g = G.random_csr(g.m, g.n, np.diff(g.row_ptr).astype(np.int32), 11)
    elif case == "evil":          # one row spanning many chunks, short rows around it
        rl = rs.randint(0, 6, size=3000).astype(np.int32)
        rl[1500] = 40000
        g = G.random_csr(3000, 60000, rl, 12)
    elif case == "empty_rows":
        rl = np.where(rs.rand(5000) < 0.8, 0, rs.randint(1, 30, size=5000)).astype(np.int32)
        g = G.random_csr(5000, 700, rl, 13)
    else:
        g = G.random_csr(300, 50, np.zeros(300, np.int32), 14)
    pin = lambda a: torch.from_numpy(a).pin_memory()
    for K, dt in ((64, torch.float32), (16, torch.float32), (32, torch.bfloat16)):
        B = G.dense_int(g.n, K, seed=K + 1)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        Bh = torch.from_numpy(B).to(dt).pin_memory()
        monkeypatch.setenv("MPS_HOST_CHUNK_BYTES", str(chunk))
        for cost in (0, 24):
            C = M.spmm_host(pin(g.row_ptr), pin(g.col_idx), pin(g.val), g.n, Bh,
                            items_per_part=cost, min_parts=1 if cost else 0)
            assert np.array_equal(C.numpy().astype(np.float64), ref), (K, dt, cost)
        monkeypatch.setenv("MPS_HOST_SERIAL", "1")
        Cs = M.spmm_host(pin(g.row_ptr), pin(g.col_idx), pin(g.val), g.n, Bh)
        monkeypatch.delenv("MPS_HOST_SERIAL")
        assert np.array_equal(Cs.numpy(), C.numpy())


@pytest.mark.parametrize("serial", [False, True])
def test_spmm_host_strided_buffers_keep_padding(monkeypatch, serial):
    """with ldc > K (a strided C_host view) the host calls write only the K
    valid columns of each row -- the padding of the caller's host matrix keeps its
    sentinel -- and with ldb > K they read only the K valid columns of B_host (the
    B_host view ends before the padding of its last row)."""
    g = G.workload("pubmed")
    A = dev(g)
    K, ldb, ldc = 64, 72, 80
    Bfull = np.full((g.n, ldb), np.nan, np.float32)
    Bfull[:, :K] = G.dense_int(g.n, K, seed=5)
    ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, Bfull[:, :K], want_bound=False)
    pin = lambda a: torch.from_numpy(a).pin_memory()
    Bh = pin(Bfull)[:, :K]                          # stride(0) = ldb > K
    if serial:
        monkeypatch.setenv("MPS_HOST_SERIAL", "1")
    for call in ("host", "host_dense"):
        Cbuf = torch.full((g.m, ldc), -7.0, dtype=torch.float32).pin_memory()
        Ch = Cbuf[:, :K]                            # stride(0) = ldc > K
        if call == "host":
            M.spmm_host(pin(g.row_ptr), pin(g.col_idx), pin(g.val), g.n, Bh, C_host=Ch)
        else:
            M.spmm_host_dense(A, Bh, C_host=Ch)
        out = Cbuf.numpy()
        assert np.all(out[:, K:] == -7.0), call         # padding untouched
        # integer-valued B with GCN-normalised A: within the north-star tolerance
        bnd = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, np.abs(Bfull[:, :K]),
                             want_bound=False)
        r = O.check(out[:, :K], ref, bnd)
        assert r["ok"], (call, r)


@pytest.mark.parametrize("fixup", ["atomic", "carry"])
def test_spmm_host_dense_graph_resident(fixup):
    g = G.workload("pubmed")
    A = dev(g)
    for K, dt in ((64, torch.float32), (16, torch.bfloat16)):
        B = G.dense_int(g.n, K, seed=K)
        Bh = torch.from_numpy(B).to(dt).pin_memory()
        Ci = M.CSR.from_numpy(g.row_ptr, g.col_idx, G.values_int(g.nnz, 3), g.n)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, G.values_int(g.nnz, 3), B, want_bound=False)
        C = M.spmm_host_dense(Ci, Bh, fixup=fixup)
        assert np.array_equal(C.numpy().astype(np.float64), ref)
    Bf = G.features("pubmed", 64)
    ref, bnd = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, Bf)
    C = M.spmm_host_dense(A, torch.from_numpy(Bf).pin_memory(), fixup=fixup)
    assert O.check(C.numpy(), ref, bnd)["ok"]


# --------------------------------------------------------------------------------
# a6: sharding, loopback on one GPU (every rank run in turn, tails gathered by copy)
# --------------------------------------------------------------------------------
@pytest.mark.parametrize("fixup", ["atomic", "carry"])
def test_sharded_loopback_exact(fixup):
    rs = np.random.RandomState(12)
    graphs = [rand_graph(rs, 300, 100, 10, seed=s) for s in range(4)]
    rl = np.ones(50, np.int32)
    rl[20] = 5000                                       # one row spanning 3+ shards
    graphs.append(G.random_csr(50, 100, rl, 9))
    graphs.append(G.workload("cora", values="int"))
    for g in graphs:
        K = 24
        B = G.dense_int(g.n, K, seed=4)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        for world in (1, 2, 3, 4, 8):
            shards = [M.ShardedSpMM(g.row_ptr, g.col_idx, g.val, g.n, K, r, world, "cuda",
                                    fixup=fixup, items_per_part=7, min_parts=1)
                      for r in range(world)]
            X, Y, T = shards[0].X, shards[0].Y, shards[0].T
            ox, oy, ot = O.shard(g.row_ptr, world)
            assert np.array_equal(X, ox) and np.array_equal(Y, oy) and np.array_equal(T, ot)
            Bt = tB(B)
            for s in shards:
                s.local(Bt)
            tails = torch.cat([s.tail for s in shards])
            out = np.zeros_like(ref)
            for r, s in enumerate(shards):
                # local result before the exchange equals the oracle's shard_local
                Cl, tail = O.shard_local(g.row_ptr, g.col_idx, g.val, B, X, Y, r)
                assert np.array_equal(s.tail.cpu().numpy().astype(np.float64), tail)
                Cr = s.settle(tails).cpu().numpy().astype(np.float64)
                out[X[r]:X[r + 1]] = Cr
            assert np.array_equal(out, ref), (world, fixup)


# --------------------------------------------------------------------------------
# full-size BASELINE workloads: sampled rows + whole-matrix properties
# --------------------------------------------------------------------------------
def _sampled_check(g, K, fixup, cost=0, dtype=torch.float32, seed=0):
    B = G.features(g.name, K)
    Bt = tB(B, dtype)
    if dtype == torch.bfloat16:
        B = Bt.float().cpu().numpy()
    A = dev(g)
    sch = M.Schedule.build(A, K, b_dtype=dtype, items_per_part=cost)
    C = torch.full((g.m, K), float("nan"), device="cuda")
    M.spmm(A, Bt, schedule=sch, fixup=fixup, out=C)
    torch.cuda.synchronize()
    assert not torch.isnan(C).any()
    cx = sch.coord_x.cpu().numpy()
    cy = sch.coord_y.cpu().numpy()
    split = cx[(cx < g.m) & (cy > g.row_ptr[np.minimum(cx, g.m)])]
    deg = np.diff(g.row_ptr)
    rs = np.random.RandomState(seed)
    rows = np.unique(np.concatenate([
        rs.choice(g.m, 3000), split[rs.choice(len(split), min(len(split), 2000))] if len(split) else [],
        np.argsort(deg)[-50:], [0, g.m - 1]]).astype(np.int64))
    ref, bnd = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, rows=rows)
    r = O.check(C[torch.from_numpy(rows).cuda()].cpu().numpy(), ref, bnd)
    assert r["ok"], r
    # whole matrix: sum_i C[i,:] = w^T B with w[c] = sum of A's column c (fp64, any size)
    w = np.bincount(g.col_idx, weights=g.val.astype(np.float64), minlength=g.n)
    colsum_ref = w @ B.astype(np.float64)
    colsum_abs = np.abs(w) @ np.abs(B.astype(np.float64))
    colsum = C.double().sum(0).cpu().numpy()
    assert np.all(np.abs(colsum - colsum_ref) <= 1e-5 * colsum_abs + 1e-3)
    return sch


@pytest.mark.slow
@pytest.mark.parametrize("fixup", ["atomic", "carry"])
def test_rmat_full_size(fixup):
    g = G.workload("rmat")
    _sampled_check(g, 64, fixup)


@pytest.mark.slow
def test_reddit_full_size_k64_and_k256():
    g = G.workload("reddit")
    _sampled_check(g, 64, "atomic")
    _sampled_check(g, 256, "atomic")
    _sampled_check(g, 64, "carry")


@pytest.mark.slow
def test_products_full_size_k128():
    g = G.workload("products")
    _sampled_check(g, 128, "atomic")
    _sampled_check(g, 128, "atomic", dtype=torch.bfloat16)


@pytest.mark.gpu
@pytest.mark.parametrize("wl,K", [("cora", 16), ("rmat", 64)])
def test_bench_cuda_graph_replays_the_step(wl, K):
    """bench.py --cuda-graph: the captured graph must hold the step's launches (the bench
    itself replays once against the eager result and raises on a mismatch), and a replay
    cannot be faster than the segment kernel's share of the eager step."""
    import json, os, subprocess, sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    base = [sys.executable, os.path.join(root, "bench.py"), "--workload", wl, "--K", str(K),
            "--steps", "5", "--warmup", "3", "--e2e-steps", "0", "--no-cpu-baseline",
            "--no-cusparse", "--no-l2-probe"]
    lines = {}
    for mode in ("eager", "graph"):
        cmd = base + (["--cuda-graph"] if mode == "graph" else [])
        r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=root)
        assert r.returncode == 0, r.stderr[-2000:]
        lines[mode] = json.loads([ln for ln in r.stdout.splitlines() if ln.startswith("{")][-1])
    assert lines["graph"]["config"]["cuda_graph"] is True
    # the eager step's segment kernel alone bounds the graph replay from below (its
    # fastest eager step: on tiny graphs one slow step inflates the eager mean)
    eager = lines["eager"]
    floor = min(eager["segment_ms"], eager["step_ms_min_median"][0])
    assert lines["graph"]["ms_per_step"] >= 0.5 * floor
