"""CPU fp64 oracle for MergePath-SpMM -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product package
(``paper_conf_ispass_shangndk23_b200``) never imports it, and the two share no code:
the arithmetic lives in ``oracle/oracle.c`` (plain C, fp64, built with gcc), this file
only marshals numpy arrays through ctypes.  Every function cites the passage of the
paper (``/root/reference/PAPER.md`` line, "P:<line>") that it follows; the pins that
check it against something other than itself are in ``tests/test_oracle_pins.py``.

O8 (``check``) is the north-star tolerance |C - C_ref| <= 1e-5 * (|A||B|) + 1e-7.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

_i64 = ctypes.c_int64
_i32 = ctypes.c_int32
_p = ctypes.c_void_p


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (-O2, OpenMP, no fp contraction)."""
    if (not force and os.path.exists(_LIB_PATH)
            and os.path.getmtime(_LIB_PATH) >= os.path.getmtime(_SRC)):
        return _LIB_PATH
    tmp = _LIB_PATH + ".tmp%d" % os.getpid()
    cmd = ["gcc", "-std=c99", "-O2", "-fopenmp", "-ffp-contract=off", "-fPIC", "-shared",
           _SRC, "-o", tmp, "-lm"]
    subprocess.check_call(cmd)
    os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def _L():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        lib.oracle_csr_spmm_f64.argtypes = [_i64, _p, _p, _p, _p, _i64, _i32, _p, _i64, _p, _p, _i64]
        lib.oracle_dense_spmm_f64.argtypes = [_i64, _i64, _p, _p, _p, _p, _i64, _i32, _p, _i64]
        lib.oracle_plan.argtypes = [_i64, _i64, _i64, _i64, _p, _p]
        lib.oracle_merge_coord.argtypes = [_p, _i64, _i64, _i64, _p, _p]
        lib.oracle_partition.argtypes = [_p, _i64, _i64, _i64, _i64, _i64, _i64, _p, _p]
        lib.oracle_merge_coord64.argtypes = [_p, _i64, _i64, _i64, _p, _p]
        lib.oracle_partition64.argtypes = [_p, _i64, _i64, _i64, _i64, _i64, _i64, _p, _p]
        lib.oracle_merge_walk.argtypes = [_p, _i64, _i64, _p, _p]
        lib.oracle_alg2_emulate.argtypes = [_i64, _p, _p, _p, _p, _i64, _i32, _p, _p, _i64,
                                            _p, _i64, _p, _p]
        lib.oracle_shard.argtypes = [_p, _i64, _i64, _i32, _p, _p, _p]
        lib.oracle_xw_f64.argtypes = [_i64, _i64, _i32, _p, _i64, _p, _i64, _i32, _p, _i64]
        lib.oracle_shard_local.argtypes = [_i64, _p, _p, _p, _p, _i64, _i32, _i64, _i64, _i64,
                                           _i64, _p, _i64, _p]
        _lib = lib
    return _lib


def _ptr(a):
    return a.ctypes.data_as(ctypes.c_void_p) if a is not None and a.size else None


def _c(a, dt):
    return np.ascontiguousarray(a, dtype=dt)


def num_threads() -> int:
    return int(_L().oracle_num_threads())


def csr_spmm_f64(row_ptr, col_idx, val, B, K=None, rows=None, want_bound=True):
    """O1 + O2 (sec. II): C = A*B and Bnd = |A|*|B| in fp64.

    ``B`` is a 2-D float32 array (row-major, leading dimension = B.shape[1]);
    ``rows`` (optional) restricts the output to those rows, in that order.
    """
    rp, ci, av = _c(row_ptr, np.int32), _c(col_idx, np.int32), _c(val, np.float32)
    B = np.ascontiguousarray(B, dtype=np.float32)
    m = rp.shape[0] - 1
    K = B.shape[1] if K is None else K
    rws = None if rows is None else _c(rows, np.int64)
    count = m if rws is None else rws.shape[0]
    C = np.zeros((count, K), np.float64)
    bnd = np.zeros((count, K), np.float64) if want_bound else None
    rc = _L().oracle_csr_spmm_f64(m, _ptr(rp), _ptr(ci), _ptr(av), _ptr(B), B.shape[1], K,
                                  _ptr(rws), count, _ptr(C), _ptr(bnd), K)
    assert rc == 0
    return (C, bnd) if want_bound else C


def dense_spmm_f64(row_ptr, col_idx, val, n_cols, B):
    """O3: materialise A densely (duplicates summed), then the triple loop."""
    rp, ci, av = _c(row_ptr, np.int32), _c(col_idx, np.int32), _c(val, np.float32)
    B = np.ascontiguousarray(B, dtype=np.float32)
    m, K = rp.shape[0] - 1, B.shape[1]
    C = np.zeros((m, K), np.float64)
    rc = _L().oracle_dense_spmm_f64(m, n_cols, _ptr(rp), _ptr(ci), _ptr(av), _ptr(B),
                                    B.shape[1], K, _ptr(C), K)
    assert rc == 0
    return C


def plan(m, nnz, cost, min_parts):
    """O4a: Alg. 1 lines 2-3 + sec. III-C thread count."""
    P, L = ctypes.c_int64(), ctypes.c_int64()
    rc = _L().oracle_plan(m, nnz, cost, min_parts, ctypes.byref(P), ctypes.byref(L))
    if rc != 0:
        raise ValueError("invalid plan arguments")
    return P.value, L.value


def merge_coord(row_ptr, d):
    """O4b: BINARYSEARCH of Alg. 1 lines 6-7 (Fig. 3 text P:96)."""
    rp = _c(row_ptr, np.int32)
    m = rp.shape[0] - 1
    x, y = ctypes.c_int64(), ctypes.c_int64()
    rc = _L().oracle_merge_coord(_ptr(rp), m, int(rp[-1]), d, ctypes.byref(x), ctypes.byref(y))
    if rc != 0:
        raise ValueError("diagonal out of range")
    return x.value, y.value


def partition(row_ptr, num_parts, items_per_part, diag_begin=0, diag_end=None):
    """O4c: coordinates of diagonals d_p = begin + min(p*L, end-begin), p = 0..P."""
    rp = _c(row_ptr, np.int32)
    m, nnz = rp.shape[0] - 1, int(rp[-1])
    diag_end = m + nnz if diag_end is None else diag_end
    cx = np.zeros(num_parts + 1, np.int32)
    cy = np.zeros(num_parts + 1, np.int32)
    rc = _L().oracle_partition(_ptr(rp), m, nnz, diag_begin, diag_end, num_parts,
                               items_per_part, _ptr(cx), _ptr(cy))
    if rc != 0:
        raise ValueError("invalid partition arguments")
    return cx, cy


def partition64(row_ptr, num_parts, items_per_part, diag_begin=0, diag_end=None):
    """O4c with int64 row offsets (NEXT-4): (cx int32[P+1], cy int64[P+1])."""
    rp = _c(row_ptr, np.int64)
    m, nnz = rp.shape[0] - 1, int(rp[-1])
    diag_end = m + nnz if diag_end is None else diag_end
    cx = np.zeros(num_parts + 1, np.int32)
    cy = np.zeros(num_parts + 1, np.int64)
    rc = _L().oracle_partition64(_ptr(rp), m, nnz, diag_begin, diag_end, num_parts,
                                 items_per_part, _ptr(cx), _ptr(cy))
    if rc != 0:
        raise ValueError("invalid partition arguments")
    return cx, cy


def merge_walk(row_ptr):
    """O5: the explicit merge of row ends and non-zeros."""
    rp = _c(row_ptr, np.int32)
    m, nnz = rp.shape[0] - 1, int(rp[-1])
    xs = np.zeros(m + nnz + 1, np.int32)
    ys = np.zeros(m + nnz + 1, np.int32)
    _L().oracle_merge_walk(_ptr(rp), m, nnz, _ptr(xs), _ptr(ys))
    return xs, ys


def alg2_emulate(row_ptr, col_idx, val, B, cx, cy, C_init=None):
    """O6: serial Alg. 2 in fp64 with (#atomic, #regular) counters."""
    rp, ci, av = _c(row_ptr, np.int32), _c(col_idx, np.int32), _c(val, np.float32)
    B = np.ascontiguousarray(B, dtype=np.float32)
    cx, cy = _c(cx, np.int32), _c(cy, np.int32)
    m, K = rp.shape[0] - 1, B.shape[1]
    C = np.zeros((m, K), np.float64) if C_init is None else np.array(C_init, np.float64)
    na, nr = ctypes.c_int64(), ctypes.c_int64()
    rc = _L().oracle_alg2_emulate(m, _ptr(rp), _ptr(ci), _ptr(av), _ptr(B), B.shape[1], K,
                                  _ptr(cx), _ptr(cy), cx.shape[0] - 1, _ptr(C), K,
                                  ctypes.byref(na), ctypes.byref(nr))
    assert rc == 0
    return C, na.value, nr.value


def shard(row_ptr, world):
    """O7: merge-path shard bounds (X, Y) and tail rows (north-star stage 4)."""
    rp = _c(row_ptr, np.int32)
    m, nnz = rp.shape[0] - 1, int(rp[-1])
    X = np.zeros(world + 1, np.int32)
    Y = np.zeros(world + 1, np.int32)
    T = np.zeros(world, np.int32)
    rc = _L().oracle_shard(_ptr(rp), m, nnz, world, _ptr(X), _ptr(Y), _ptr(T))
    assert rc == 0
    return X, Y, T


def shard_local(row_ptr, col_idx, val, B, X, Y, g):
    """O7b: shard g's owned rows [X_g, X_{g+1}) and tail vector, plain fp64 sums."""
    rp, ci, av = _c(row_ptr, np.int32), _c(col_idx, np.int32), _c(val, np.float32)
    B = np.ascontiguousarray(B, dtype=np.float32)
    m, K = rp.shape[0] - 1, B.shape[1]
    rows = int(X[g + 1]) - int(X[g])
    C = np.zeros((max(rows, 0), K), np.float64)
    tail = np.zeros(K, np.float64)
    _L().oracle_shard_local(m, _ptr(rp), _ptr(ci), _ptr(av), _ptr(B), B.shape[1], K,
                            int(X[g]), int(Y[g]), int(X[g + 1]), int(Y[g + 1]),
                            _ptr(C) if C.size else None, K, _ptr(tail) if K else None)
    return C, tail


def xw_f64(X, W, relu=False):
    """O9 (sec. II: H' = sigma(A X W)): the combination X*W of a GCN layer, and
    the ReLU when ``relu``, in fp64.  X: n x F, W: F x N (W itself, not its transpose),
    any float dtype convertible to float32 exactly (bf16 values are)."""
    X = np.ascontiguousarray(X, dtype=np.float32)
    W = np.ascontiguousarray(W, dtype=np.float32)
    n, F = X.shape
    F2, N = W.shape
    assert F == F2
    out = np.zeros((n, N), np.float64)
    rc = _L().oracle_xw_f64(n, F, N, _ptr(X), F, _ptr(W), N, 1 if relu else 0,
                            _ptr(out), N)
    assert rc == 0
    return out


def check(C, C_ref, bound, rel=1e-5, abs_tol=1e-7):
    """O8: north-star tolerance |C - C_ref| <= rel*(|A||B|) + abs, element-wise.

    Returns a dict with the worst ratio err / allowed, the violation count and the
    NaN/Inf count; ``ok`` is True iff there are no violations and no NaN/Inf.
    """
    C = np.asarray(C, np.float64)
    C_ref = np.asarray(C_ref, np.float64)
    allowed = rel * np.asarray(bound, np.float64) + abs_tol
    bad_nf = int(np.count_nonzero(~np.isfinite(C)))
    err = np.abs(C - C_ref)
    err = np.where(np.isfinite(err), err, np.inf)
    ratio = err / allowed
    viol = int(np.count_nonzero(ratio > 1.0))
    worst = float(ratio.max()) if ratio.size else 0.0
    return {"ok": viol == 0 and bad_nf == 0, "worst_ratio": worst, "violations": viol,
            "nonfinite": bad_nf}
