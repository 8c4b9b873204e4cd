"""The seeded input generators produce the recipe DESIGN.md states (CPU only)."""
import numpy as np
import pytest

import graphgen as G


@pytest.mark.parametrize("name,n,nnz", [("cora", 2708, 10556), ("pubmed", 19717, 88648)])
def test_chung_lu_shape_and_structure(name, n, nnz):
    g = G.workload(name)
    assert (g.m, g.n, g.nnz) == (n, n, nnz)
    rp, ci = g.row_ptr, g.col_idx
    assert rp[0] == 0 and np.all(np.diff(rp) >= 0)
    rows = np.repeat(np.arange(g.m), np.diff(rp))
    assert np.all(ci >= 0) and np.all(ci < n)
    assert not np.any(rows == ci)                                  # no self loops
    # canonical CSR: strictly increasing columns inside every row
    same_row = rows[1:] == rows[:-1]
    assert np.all(ci[1:][same_row] > ci[:-1][same_row])
    # symmetric
    a = set(zip(rows.tolist(), ci.tolist()))
    assert all((c, r) in a for (r, c) in a)
    # power-law skew: max degree far above the mean
    d = np.diff(rp)
    assert d.max() > 20 * d.mean()
    # GCN values 1/sqrt(d_i d_j)
    np.testing.assert_allclose(g.val, 1.0 / np.sqrt(d[rows] * d[ci].astype(np.float64)),
                               rtol=1e-6)


def test_deterministic():
    a, b = G.workload("cora"), G.workload("cora")
    assert a.digest() == b.digest() and np.array_equal(a.val, b.val)
    assert np.array_equal(G.features("cora", 16), G.features("cora", 16))
    assert not np.array_equal(G.features("cora", 16), G.features("cora", 16, seed=9))


def test_dense_ranges():
    B = G.dense_uniform(1000, 33, seed=1)
    assert B.min() >= -1.0 and B.max() < 1.0 and abs(B.mean()) < 0.02
    Bi = G.dense_int(1000, 33, seed=1)
    assert set(np.unique(Bi).tolist()) <= set(range(-4, 5))
    Bp = G.dense_uniform(10, 5, seed=1, ld=8)
    assert np.all(Bp[:, 5:] == 0) and np.array_equal(Bp[:, :5], G.dense_uniform(10, 5, seed=1))


def test_random_csr_adversarial():
    rl = np.array([0, 5, 0, 0, 9, 1], np.int32)
    g = G.random_csr(6, 4, rl, seed=3, canonical=False)
    assert np.array_equal(np.diff(g.row_ptr), rl)
    assert set(np.unique(g.val).tolist()) <= {1.0, 2.0, 3.0}


def test_wide_generator_host_equals_device_formula():
    """NEXT-4 wide graphs: the numpy (host) and torch (device) evaluations of the
    counter-based hash give the same bytes; splitmix64's first output from state 0 is
    the published 0xE220A8397B1DCDAF."""
    import torch
    assert int(G._mix_np(np.uint64(0))) == 0xE220A8397B1DCDAF
    j = np.arange(0, 100000, dtype=np.int64) * 104729 + (1 << 31) - 5
    c, v = G.wide_cols_vals_host(j, 999983, 11)
    ct, vt = G.wide_cols_vals_device(0, 999983, 11, device="cpu")  # empty, exercises the API
    assert ct.numel() == 0
    jt = torch.from_numpy(j)
    assert np.array_equal(c, (G._h31_torch(12, jt) % 999983).to(torch.int32).numpy())
    assert np.array_equal(v, (1 + G._h31_torch(13, jt) % 3).to(torch.float32).numpy())
    assert c.min() >= 0 and c.max() < 999983 and set(np.unique(v)) == {1.0, 2.0, 3.0}
    rp = G.wide_row_ptr(1000, 2048, 3, evil=[(7, 10 ** 6)])
    assert rp.dtype == np.int64 and rp[0] == 0 and np.all(np.diff(rp) >= 0)
    assert rp[8] - rp[7] == 10 ** 6 and np.diff(rp).max() == 10 ** 6
