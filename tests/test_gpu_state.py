"""The library keeps no state between calls (include/mpspmm.h "Ownership").

The segment kernel's dynamic claim counters live in the caller's workspace, so two
captured CUDA graphs -- captured more than a thousand library launches apart, replayed
concurrently on two streams -- each own their counters and both reproduce the oracle
bit-exactly (integer-valued inputs make every summation order exact).  With a
process-wide counter ring they would collide after wrap-around and skip or repeat
segments.
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


def _graph(seed, m=150_000, n=60_000):
    rs = np.random.RandomState(seed)
    rl = rs.geometric(1.0 / 12, size=m).astype(np.int32)   # short, skewed rows
    rl[rs.randint(m, size=4)] = 20_000                      # evil rows
    return G.random_csr(m, n, rl, seed, values="int")


def _capture(step, B):
    step(B)                                   # outside capture (occupancy queries)
    torch.cuda.synchronize()
    cg = torch.cuda.CUDAGraph()
    with torch.cuda.graph(cg):
        step(B)
    return cg


def test_two_graphs_captured_far_apart_replay_concurrently():
    K = 64
    g1, g2 = _graph(1), _graph(2)
    B1, B2 = G.dense_int(g1.n, K, seed=1), G.dense_int(g2.n, K, seed=2)
    ref1 = O.csr_spmm_f64(g1.row_ptr, g1.col_idx, g1.val, B1, want_bound=False)
    ref2 = O.csr_spmm_f64(g2.row_ptr, g2.col_idx, g2.val, B2, want_bound=False)
    A1 = M.CSR.from_numpy(g1.row_ptr, g1.col_idx, g1.val, g1.n)
    A2 = M.CSR.from_numpy(g2.row_ptr, g2.col_idx, g2.val, g2.n)
    B1t, B2t = torch.from_numpy(B1).cuda(), torch.from_numpy(B2).cuda()
    s1 = M.OnlineStep(A1, K, items_per_part=64)
    s2 = M.OnlineStep(A2, K, items_per_part=64)
    # long enough schedules for dynamic segment claims (the counters under test)
    assert s1.P >= 4 * 2 * 8 * torch.cuda.get_device_properties(0).multi_processor_count
    cg1 = _capture(s1, B1t)
    # > 1024 library launches between the two captures
    filler = M.OnlineStep(A1, K, items_per_part=64)
    for _ in range(600):
        filler(B1t)
    torch.cuda.synchronize()
    cg2 = _capture(s2, B2t)
    st_a, st_b = torch.cuda.Stream(), torch.cuda.Stream()
    for rep in range(3):
        s1.C.fill_(float("nan"))
        s2.C.fill_(float("nan"))
        torch.cuda.synchronize()
        for _ in range(4):                    # overlapping replays on two streams
            with torch.cuda.stream(st_a):
                cg1.replay()
            with torch.cuda.stream(st_b):
                cg2.replay()
        torch.cuda.synchronize()
        assert np.array_equal(s1.C.cpu().numpy().astype(np.float64), ref1), rep
        assert np.array_equal(s2.C.cpu().numpy().astype(np.float64), ref2), rep


def test_offline_segments_reuse_workspace_counters():
    """mps_spmm_segments zeroes its workspace's claim counters itself: garbage in the
    workspace on entry, and many back-to-back calls, give the same exact result."""
    K = 32
    g = _graph(3)
    B = G.dense_int(g.n, K, seed=3)
    ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
    A = M.CSR.from_numpy(g.row_ptr, g.col_idx, g.val, g.n)
    st = M.OnlineStep(A, K, items_per_part=32)
    st.ws.fill_(0xA5)                         # garbage claim counters
    Bt = torch.from_numpy(B).cuda()
    for _ in range(20):
        st(Bt)
    torch.cuda.synchronize()
    assert np.array_equal(st.C.cpu().numpy().astype(np.float64), ref)
