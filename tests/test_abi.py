"""The C-ABI library loads on a GPU-less host and exports every symbol that
include/mpspmm.h declares; host-only entry points (plan, shard bounds) agree with the
oracle and report errors through status codes.  No device compute here."""
import ctypes
import os
import re

import numpy as np
import pytest

import graphgen as G
import oracle as O
import paper_conf_ispass_shangndk23_b200 as M
from paper_conf_ispass_shangndk23_b200 import _lib

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    with open(os.path.join(ROOT, "include", "mpspmm.h")) as f:
        src = f.read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(mps_[a-z_0-9]+)\s*\(", src)))


def test_header_symbols_exported():
    names = declared_functions()
    assert len(names) >= 17
    lib = ctypes.CDLL(_lib.LIB_PATH)
    for n in names:
        assert hasattr(lib, n), n
        assert n in _lib.EXPORTED, n     # and bound one-to-one in Python
    assert set(_lib.EXPORTED) == set(names)


def test_abi_version_and_status_strings():
    assert M.mps_abi_version() == 2
    assert M.mps_status_string(0) == b"MPS_OK"
    assert M.mps_status_string(4) == b"MPS_ERR_WORKSPACE"


def test_plan_matches_oracle():
    rs = np.random.RandomState(0)
    for _ in range(500):
        m, nnz = int(rs.randint(0, 10 ** 7)), int(rs.randint(0, 10 ** 8))
        cost, pmin = int(rs.randint(1, 5000)), int(rs.randint(1, 20000))
        assert M.plan(m, nnz, 64, 0, cost, pmin) == O.plan(m, nnz, cost, pmin)
    P, L = M.plan(232965, 114615892, 64)          # library defaults
    assert P * L >= 232965 + 114615892


def test_plan_errors():
    P, L = ctypes.c_int64(), ctypes.c_int64()
    with pytest.raises(M.MpsError) as e:
        M.mps_plan(1, 1, 8, 9, 0, 0, ctypes.byref(P), ctypes.byref(L))
    assert e.value.status == M.MPS_ERR_UNSUPPORTED
    with pytest.raises(M.MpsError) as e:
        M.mps_plan(2 ** 31, 0, 8, 0, 0, 0, ctypes.byref(P), ctypes.byref(L))
    assert e.value.status == M.MPS_ERR_UNSUPPORTED
    with pytest.raises(M.MpsError) as e:
        M.mps_plan(-1, 0, 8, 0, 0, 0, ctypes.byref(P), ctypes.byref(L))
    assert e.value.status == M.MPS_ERR_INVALID
    with pytest.raises(M.MpsError) as e:
        M.mps_spmm_online(None, None, 0, 8, 8, None, 8, 0, 0, 1, None, 0, None)
    assert e.value.status == M.MPS_ERR_INVALID


@pytest.mark.parametrize("world", [1, 2, 3, 4, 8, 64])
def test_shard_bounds_match_oracle(world):
    for name in ("cora", "pubmed"):
        g = G.workload(name)
        X, Y, T = M.shard_bounds(g.row_ptr, world)
        ox, oy, ot = O.shard(g.row_ptr, world)
        assert np.array_equal(X, ox) and np.array_equal(Y, oy) and np.array_equal(T, ot)
    rl = np.zeros(9, np.int32)
    rl[4] = 1000
    g = G.random_csr(9, 9, rl, 1)
    X, Y, T = M.shard_bounds(g.row_ptr, world)
    assert np.array_equal(T, O.shard(g.row_ptr, world)[2])


def test_plan64_host_only():
    """NEXT-4: mps_plan64 lifts the 2^31 limit on M = m + nnz (same Alg. 1 sizing as
    the oracle); m >= 2^31 stays unsupported (rows are int32)."""
    for (m, nnz, cost, pmin) in [(10, 2 ** 31, 2048, 1), (2 ** 31 - 1, 2 ** 40, 4096, 1184),
                                 (5, 0, 7, 1), (232965, 114615892, 2048, 1184)]:
        assert M.plan(m, nnz, 64, 0, cost, pmin, wide=True) == O.plan(m, nnz, cost, pmin)
    P, L = ctypes.c_int64(), ctypes.c_int64()
    with pytest.raises(M.MpsError) as e:
        M.mps_plan64(2 ** 31, 0, 8, 0, 0, 0, ctypes.byref(P), ctypes.byref(L))
    assert e.value.status == M.MPS_ERR_UNSUPPORTED
    a = M.mps_csr64(2 ** 31, 4, 0, None, None, None)
    nb = ctypes.c_size_t()
    with pytest.raises(M.MpsError) as e:
        M.mps_spmm64_online_workspace_bytes(ctypes.byref(a), 16, 0, 0, 0, 1, ctypes.byref(nb))
    assert e.value.status == M.MPS_ERR_UNSUPPORTED
    a = M.mps_csr64(1000, 1000, 3 * 2 ** 30, None, None, None)
    M.mps_spmm64_online_workspace_bytes(ctypes.byref(a), 16, 0, 0, 0, 1, ctypes.byref(nb))
    Pp, Lp = M.plan(1000, 3 * 2 ** 30, 16, 0, 0, 0, wide=True)
    assert nb.value >= (Pp + 1) * 12       # int32 coord_x + int64 coord_y


def test_shard_bounds64_host_only():
    """NEXT-4 scale-out: mps_shard_bounds64 is the Alg. 1 closed form at G diagonals
    (oracle O4-64 with P = G, L = ceil(M/G)) on a 5e9-non-zero row_ptr; tails by R24."""
    rs = np.random.RandomState(3)
    m = 300_000
    rl = rs.randint(0, 30_000, size=m).astype(np.int64)
    rl[rs.randint(m, size=2)] = 10 ** 9
    rp = np.zeros(m + 1, np.int64)
    np.cumsum(rl, out=rp[1:])
    nnz = int(rp[-1])
    for G_ in (1, 2, 3, 8, 16):
        X, Y, T = M.shard_bounds(rp, G_)
        assert Y.dtype == np.int64
        ox, oy = O.partition64(rp, G_, -(-(m + nnz) // G_))
        assert np.array_equal(X, ox) and np.array_equal(Y, oy)
        for g in range(G_):
            r = X[g + 1]
            assert T[g] == (r if (r < m and Y[g + 1] > rp[r]) else -1)
    # the int32 form agrees with the int64 one where both apply
    g = G.random_csr(500, 300, np.random.RandomState(0).randint(0, 20, 500).astype(np.int32), 1)
    X32, Y32, T32 = M.shard_bounds(g.row_ptr, 8)
    X64, Y64, T64 = M.shard_bounds(g.row_ptr.astype(np.int64), 8)
    assert np.array_equal(X32, X64) and np.array_equal(Y32, Y64) and np.array_equal(T32, T64)


def test_multi_gpu_entry_points_validate_before_touching_the_gpu():
    """Argument checks of the peer-memory entry points return status codes on a host
    without a GPU (no device call is reached)."""
    assert M.mps_signal_bytes() == 64 * 16 * 4
    assert M.mps_shard_mailbox_bytes(128) >= 256 + 2 * 16 * 128 * 4
    assert M.mps_shard_mailbox_bytes(128) % 256 == 0
    arr = (ctypes.c_void_p * 2)(None, None)
    for call in (lambda: M.mps_peer_signal(None, 2, 0, 0, 1, None),
                 lambda: M.mps_peer_signal(arr, 2, 0, 0, 1, None),          # NULL buffers
                 lambda: M.mps_peer_signal(arr, 17, 0, 0, 1, None),         # world > 16
                 lambda: M.mps_peer_signal(arr, 2, 2, 0, 1, None),          # rank >= world
                 lambda: M.mps_peer_signal(arr, 2, 0, 64, 1, None),         # slot >= 64
                 lambda: M.mps_peer_wait(None, 2, 0, 1, None),
                 lambda: M.mps_peer_wait(ctypes.c_void_p(16), 2, 0, 0, None)):  # epoch 0
        with pytest.raises(M.MpsError) as e:
            call()
        assert e.value.status == M.MPS_ERR_INVALID
    a = M.mps_csr(10, 10, 0, None, None, None)
    X = np.zeros(3, np.int32)
    with pytest.raises(M.MpsError) as e:        # p2p exchange needs the mailbox array
        M.mps_spmm_shard_p2p(ctypes.byref(a), None, 0, 8, 8, X.ctypes.data_as(ctypes.c_void_p),
                             X.ctypes.data_as(ctypes.c_void_p), X.ctypes.data_as(ctypes.c_void_p),
                             0, 2, 0, 0, None, 8, None, 1, None, 1, None, 0, None)
    assert e.value.status == M.MPS_ERR_INVALID
    with pytest.raises(M.MpsError) as e:        # more than 16 destinations
        dst = (ctypes.c_void_p * 17)(*([16] * 17))
        M.mps_xw_bf16_bcast(ctypes.c_void_p(16), 10, 64, 64, ctypes.c_void_p(16), 32, 64, dst,
                            17, 0, 32, None)
    assert e.value.status in (M.MPS_ERR_INVALID, M.MPS_ERR_UNSUPPORTED)
