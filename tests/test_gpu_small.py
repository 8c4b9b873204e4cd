"""The one-launch online path for small graphs (small.cu, MPS_PATH_SMALL_FUSED): every CTA
stages row_ptr in shared memory, every warp computes its own merge-path coordinates
(Alg. 1 lines 6-7), walks its segment (Alg. 2) and leaves the cut
rows' pieces to the carry reduction.

Bars: the coordinates it publishes equal the oracle's O4 bit-exactly; integer-valued
inputs give C == O1 bit-exactly (every fp32 sum is exact); float inputs are within the
north-star tolerance (O8); NaN-prefilled C leaves no NaN; ReLU epilogue; misaligned B.
"""
import ctypes

import numpy as np
import pytest
import torch

import graphgen as G
import oracle as O

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_ispass_shangndk23_b200 as M


def _graph(rs, m, n, kind, seed):
    if kind == 0:
        rl = rs.randint(0, 9, size=m)
    elif kind == 1:                                   # mostly empty rows
        rl = np.where(rs.rand(m) < 0.7, 0, rs.randint(1, 6, size=m))
    elif kind == 2:                                   # one evil row spanning many segments
        rl = rs.randint(0, 3, size=m)
        rl[rs.randint(m)] = min(n, 1500)
    else:                                             # long first and last rows
        rl = rs.randint(0, 5, size=m)
        rl[0] = rl[-1] = min(n, 700)
    return G.random_csr(m, n, rl.astype(np.int32), seed, values="int")


def _run(A, B, fixup="auto", cost=0, min_parts=0, epilogue="none", nan=True):
    st = M.OnlineStep(A, B.shape[1], b_dtype=B.dtype, fixup=fixup, items_per_part=cost,
                      min_parts=min_parts)
    if nan:
        st.C.fill_(float("nan"))
    path = st.resolve(B)
    if epilogue == "none":
        st(B)
    else:
        M.spmm(A, B, fixup=fixup, items_per_part=cost, min_parts=min_parts, out=st.C,
               epilogue=epilogue)
    torch.cuda.synchronize()
    return st, path


@pytest.mark.parametrize("K", [1, 3, 4, 8, 15, 16, 17, 32, 64, 100, 128])
def test_small_fused_integer_exact_f32(K):
    rs = np.random.RandomState(K)
    for trial in range(8):
        m = int(rs.randint(1, 2500))
        g = _graph(rs, m, 900, trial % 4, seed=trial + 10 * K)
        B = G.dense_int(900, K, seed=trial)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        A = M.CSR.from_numpy(g.row_ptr, g.col_idx, g.val, g.n)
        cost = [0, 1, 5, 12, 64, 300][trial % 6]
        st, path = _run(A, torch.from_numpy(B).cuda(), cost=cost, min_parts=1 if cost else 0)
        assert path == M.MPS_PATH_SMALL_FUSED, (K, m, cost)
        ox, oy = O.partition(g.row_ptr, st.P, st.L)
        assert np.array_equal(st.cx.cpu().numpy(), ox) and np.array_equal(st.cy.cpu().numpy(), oy)
        assert np.array_equal(st.C.cpu().numpy().astype(np.float64), ref), (K, trial, cost)


@pytest.mark.parametrize("K", [8, 16, 64, 128, 256])
def test_small_fused_integer_exact_bf16(K):
    rs = np.random.RandomState(100 + K)
    for trial in range(6):
        m = int(rs.randint(1, 2000))
        g = _graph(rs, m, 700, trial % 4, seed=trial + 7 * K)
        B = G.dense_int(700, K, seed=trial)            # |B| <= 4: exact in bf16
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        A = M.CSR.from_numpy(g.row_ptr, g.col_idx, g.val, g.n)
        st, path = _run(A, torch.from_numpy(B).cuda().to(torch.bfloat16), cost=[0, 7, 40][trial % 3],
                        min_parts=1)
        assert path == M.MPS_PATH_SMALL_FUSED
        assert np.array_equal(st.C.cpu().numpy().astype(np.float64), ref), (K, trial)


@pytest.mark.parametrize("name,K", [("cora", 16), ("pubmed", 16), ("pubmed", 64)])
def test_small_fused_workloads_tolerance(name, K):
    g = G.workload(name)
    Bh = G.features(name, K)
    ref, bnd = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, Bh)
    A = M.CSR.from_numpy(g.row_ptr, g.col_idx, g.val, g.n)
    st, path = _run(A, torch.from_numpy(Bh).cuda())
    assert path == M.MPS_PATH_SMALL_FUSED
    ox, oy = O.partition(g.row_ptr, st.P, st.L)
    assert np.array_equal(st.cx.cpu().numpy(), ox) and np.array_equal(st.cy.cpu().numpy(), oy)
    r = O.check(st.C.cpu().numpy(), ref, bnd)
    assert r["ok"], r
    # deterministic: the carry reduction sums the pieces in segment order
    C1 = st.C.clone()
    for _ in range(3):
        st(torch.from_numpy(Bh).cuda())
    torch.cuda.synchronize()
    assert torch.equal(st.C, C1)


def test_small_fused_relu_and_misaligned_B():
    rs = np.random.RandomState(5)
    g = _graph(rs, 1200, 500, 2, seed=3)
    K = 16
    B = G.dense_int(500, K + 1, seed=4)
    ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B[:, 1:], want_bound=False)
    A = M.CSR.from_numpy(g.row_ptr, g.col_idx, g.val, g.n)
    Bt = torch.from_numpy(B).cuda()[:, 1:]               # 4-byte offset: scalar lanes
    st, path = _run(A, Bt, cost=9, min_parts=1)
    assert path == M.MPS_PATH_SMALL_FUSED
    assert np.array_equal(st.C.cpu().numpy().astype(np.float64), ref)
    st2, _ = _run(A, Bt, cost=9, min_parts=1, epilogue="relu")
    assert np.array_equal(st2.C.cpu().numpy().astype(np.float64), np.maximum(ref, 0))


def test_small_fused_eligibility():
    """Large row_ptr, explicit atomic fix-up, or more than one column tile: the
    partition + segments path."""
    rs = np.random.RandomState(1)
    g = _graph(rs, 50_000, 1000, 0, seed=1)             # row_ptr 200 KB > shared memory
    A = M.CSR.from_numpy(g.row_ptr, g.col_idx, g.val, g.n)
    B = torch.zeros((g.n, 16), device="cuda")
    assert M.OnlineStep(A, 16).resolve(B) == M.MPS_PATH_PARTITION_SEGMENTS
    gs = _graph(rs, 500, 1000, 0, seed=2)
    As = M.CSR.from_numpy(gs.row_ptr, gs.col_idx, gs.val, gs.n)
    assert M.OnlineStep(As, 16, fixup="atomic").resolve(B) == M.MPS_PATH_PARTITION_SEGMENTS
    assert M.OnlineStep(As, 16, fixup="carry").resolve(B) == M.MPS_PATH_SMALL_FUSED
    B600 = torch.zeros((gs.n, 600), device="cuda")
    assert M.OnlineStep(As, 600).resolve(B600) == M.MPS_PATH_PARTITION_SEGMENTS
