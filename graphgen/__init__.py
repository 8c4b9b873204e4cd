"""Seeded synthetic inputs for MergePath-SpMM (graphs, edge values, dense B).

Used by BOTH sides of every parity check (tests, bench, smoke); holds none of the
method's arithmetic.  The arrays come from ``graphgen/gen.cpp`` (C++17/OpenMP, built with
g++), a counter-based generator, so a (recipe, seed) pair always yields the same
bytes on any machine and thread count.  The recipes follow DESIGN.md "Input recipe":
sizes and degree skew of the paper's Table II graphs and of the
BASELINE.json configs.
"""
from __future__ import annotations

import ctypes
import hashlib
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gen.cpp")
_LIB_PATH = os.path.join(_HERE, "libmpsgen.so")
_lib = None
_i64, _i32, _u64, _f64, _p = (ctypes.c_int64, ctypes.c_int32, ctypes.c_uint64,
                              ctypes.c_double, ctypes.c_void_p)


def build(force: bool = False) -> str:
    if (not force and os.path.exists(_LIB_PATH)
            and os.path.getmtime(_LIB_PATH) >= os.path.getmtime(_SRC)):
        return _LIB_PATH
    tmp = _LIB_PATH + ".tmp%d" % os.getpid()
    subprocess.check_call(["g++", "-std=c++17", "-O2", "-fopenmp", "-fPIC", "-shared", _SRC,
                           "-o", tmp])
    os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def _L():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        lib.gen_chung_lu.argtypes = [_i64, _i64, _f64, _f64, _u64]
        lib.gen_chung_lu.restype = _p
        lib.gen_rmat.argtypes = [_i32, _i64, _f64, _f64, _f64, _i32, _i64, _u64]
        lib.gen_rmat.restype = _p
        lib.gen_block_diag.argtypes = [_i64, _i64, _i64, _u64]
        lib.gen_block_diag.restype = _p
        lib.gen_random_csr.argtypes = [_i64, _i64, _p, _i32, _u64]
        lib.gen_random_csr.restype = _p
        for f in ("gen_rows", "gen_cols", "gen_nnz"):
            getattr(lib, f).argtypes = [_p]
            getattr(lib, f).restype = _i64
        lib.gen_copy.argtypes = [_p, _p, _p]
        lib.gen_free.argtypes = [_p]
        lib.gen_values_gcn.argtypes = [_i64, _p, _p, _p]
        lib.gen_values_int.argtypes = [_i64, _u64, _p]
        lib.gen_dense_uniform.argtypes = [_i64, _i32, _i64, _u64, _p]
        lib.gen_dense_int.argtypes = [_i64, _i32, _i64, _u64, _p]
        _lib = lib
    return _lib


def _ptr(a):
    return a.ctypes.data_as(ctypes.c_void_p) if a is not None and a.size else None


@dataclass
class Graph:
    """A CSR matrix A (m x n): int32 row_ptr[m+1], int32 col_idx[nnz], fp32 val[nnz]."""
    m: int
    n: int
    row_ptr: np.ndarray
    col_idx: np.ndarray
    val: np.ndarray
    name: str = ""

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1])

    def digest(self) -> str:
        h = hashlib.sha256()
        h.update(self.row_ptr.tobytes())
        h.update(self.col_idx.tobytes())
        return h.hexdigest()[:16]


def _take(h):
    lib = _L()
    m, n, nnz = lib.gen_rows(h), lib.gen_cols(h), lib.gen_nnz(h)
    rp = np.zeros(m + 1, np.int32)
    ci = np.zeros(nnz, np.int32)
    lib.gen_copy(h, _ptr(rp), _ptr(ci))
    lib.gen_free(h)
    return m, n, rp, ci


def chung_lu(n, E, alpha, dmax, seed) -> tuple:
    return _take(_L().gen_chung_lu(n, E, alpha, dmax, seed))


def block_diag(n, E, block, seed) -> tuple:
    return _take(_L().gen_block_diag(n, E, block, seed))


def rmat(scale, edge_factor, a, b, c, n_evil, evil_len, seed) -> tuple:
    return _take(_L().gen_rmat(scale, edge_factor, a, b, c, n_evil, evil_len, seed))


def random_csr(m, n, row_len, seed, canonical=True, values="int") -> Graph:
    """CSR with the given row lengths and uniformly random columns in [0, n).

    ``canonical=False`` keeps duplicate / unsorted columns (adversarial tests)."""
    rl = np.ascontiguousarray(row_len, np.int32)
    assert rl.shape[0] == m
    mm, nn, rp, ci = _take(_L().gen_random_csr(m, n, _ptr(rl), int(bool(canonical)), seed))
    g = Graph(mm, nn, rp, ci, np.zeros(ci.shape[0], np.float32), "random")
    g.val = values_int(g.nnz, seed) if values == "int" else values_gcn(g)
    return g


def values_gcn(g: Graph) -> np.ndarray:
    v = np.zeros(g.nnz, np.float32)
    _L().gen_values_gcn(g.m, _ptr(g.row_ptr), _ptr(g.col_idx), _ptr(v))
    return v


def values_int(nnz, seed) -> np.ndarray:
    v = np.zeros(nnz, np.float32)
    _L().gen_values_int(nnz, seed, _ptr(v))
    return v


def dense_uniform(rows, K, seed, ld=None) -> np.ndarray:
    ld = K if ld is None else ld
    B = np.zeros((rows, ld), np.float32)
    _L().gen_dense_uniform(rows, K, ld, seed, _ptr(B))
    return B


def dense_int(rows, K, seed, ld=None) -> np.ndarray:
    ld = K if ld is None else ld
    B = np.zeros((rows, ld), np.float32)
    _L().gen_dense_int(rows, K, ld, seed, _ptr(B))
    return B


# --------------------------------------------------------------------------------
# The five BASELINE.json workloads.
#   Chung-Lu: n nodes, E undirected edges (nnz = 2E after symmetrisation), power-law
#   weight exponent ALPHA, expected max degree dmax.  Node ids randomly permuted.
# --------------------------------------------------------------------------------
ALPHA = 0.75
WORKLOADS = {
    # name: (kind, params, seed, K list)
    "cora": ("chung_lu", dict(n=2708, E=5278, dmax=168.0), 1, (16,)),
    "pubmed": ("chung_lu", dict(n=19717, E=44324, dmax=171.0), 2, (16, 64)),
    "rmat": ("rmat", dict(scale=20, edge_factor=16, a=0.57, b=0.19, c=0.19, n_evil=8,
                          evil_len=100000), 3, (64,)),
    "reddit": ("chung_lu", dict(n=232965, E=57307946, dmax=20000.0), 4, (64, 256)),
    "products": ("chung_lu", dict(n=2449029, E=61859140, dmax=17000.0), 5, (128,)),
}


# Table II of the paper: the 22 graphs, shapes only (n, nnz, max degree).
# Type I (power-law): Chung-Lu with E = nnz//2 undirected edges and the printed max
# degree as the expected max.  Type II (structured): block-diagonal batches of small
# graphs (blocks of 32 nodes), locality preserved.  Seeds 1000 + index.
TABLE2 = [
    # (name, type, n, nnz, max_degree)
    ("Cora", 1, 2708, 10556, 168), ("Citeseer", 1, 3327, 9228, 99),
    ("Pubmed", 1, 19717, 99203, 171), ("Oregon-1", 1, 11492, 46818, 2389),
    ("As-caida", 1, 31379, 106762, 2628), ("Wiki-Vote", 1, 8297, 103689, 893),
    ("email-Enron", 1, 36692, 367662, 1383), ("email-Euall", 1, 265214, 420045, 930),
    ("Nell", 1, 65755, 251550, 4549), ("PPI", 1, 56944, 818716, 429),
    ("soc-SlashDot811", 1, 77357, 905468, 2508), ("artist", 1, 50515, 1638396, 1469),
    ("com-Amazon", 1, 334863, 1851744, 549), ("coAuthorsDBLP", 1, 299067, 1955352, 336),
    ("soc-BlogCatalog", 1, 88784, 2093195, 2538), ("amazon0601", 1, 410236, 4878874, 2760),
    ("amazon0505", 1, 403394, 5478357, 2760),
    ("PROTEINS_full", 2, 43466, 162088, 25), ("Twitter-partial", 2, 580768, 1435116, 12),
    ("DD", 2, 334925, 1686092, 19), ("Yeast", 2, 1710902, 3636546, 6),
    ("OVCAR-8H", 2, 1889542, 3946402, 5), ("SW-620H", 2, 1888584, 3944206, 5),
]
for _i, (_nm, _ty, _n, _nnz, _dmax) in enumerate(TABLE2):
    WORKLOADS["t2-" + _nm] = ("chung_lu" if _ty == 1 else "block_diag",
                              dict(n=_n, E=_nnz // 2, dmax=float(_dmax), block=32),
                              1000 + _i, (16,))


def workload(name: str, values: str = "gcn") -> Graph:
    kind, prm, seed, _ = WORKLOADS[name]
    if kind == "block_diag":
        m, n, rp, ci = block_diag(prm["n"], prm["E"], prm["block"], seed)
    elif kind == "chung_lu":
        m, n, rp, ci = chung_lu(prm["n"], prm["E"], ALPHA, prm["dmax"], seed)
    else:
        m, n, rp, ci = rmat(prm["scale"], prm["edge_factor"], prm["a"], prm["b"], prm["c"],
                            prm["n_evil"], prm["evil_len"], seed)
    g = Graph(m, n, rp, ci, np.zeros(ci.shape[0], np.float32), name)
    g.val = values_gcn(g) if values == "gcn" else values_int(g.nnz, seed)
    return g


def features(name_or_rows, K, seed=None, kind="uniform") -> np.ndarray:
    """Dense B (n x K): U[-1,1) (``uniform``) or integers in [-4, 4] (``int``)."""
    if isinstance(name_or_rows, str):
        rows = WORKLOADS[name_or_rows][1]["n"] if "n" in WORKLOADS[name_or_rows][1] else \
            1 << WORKLOADS[name_or_rows][1]["scale"]
        seed = WORKLOADS[name_or_rows][2] + 100 if seed is None else seed
    else:
        rows = int(name_or_rows)
        seed = 7 if seed is None else seed
    return dense_uniform(rows, K, seed) if kind == "uniform" else dense_int(rows, K, seed)


# --------------------------------------------------------------------------------
# NEXT-4 "wide" graphs: nnz > 2^31 (int64 row_ptr).  Too large to build on the host and
# copy per test, so the column and value arrays are a counter-based hash of the global
# non-zero index j, evaluated either on the device (torch, in chunks) or, for any
# sampled rows, on the host (numpy) -- the same bytes either way, so the oracle's inputs
# never come from the device.  splitmix64 finaliser (Steele et al.), logical shifts
# emulated on torch's signed int64.
# --------------------------------------------------------------------------------
_SM_C = (0x9E3779B97F4A7C15, 0xBF58476D1CE4E5B9, 0x94D049BB133111EB)


def _s64(c):
    return c - (1 << 64) if c >= (1 << 63) else c


def _mix_np(x):
    x = np.asarray(x, np.uint64)
    with np.errstate(over="ignore"):
        z = x + np.uint64(_SM_C[0])
        z = (z ^ (z >> np.uint64(30))) * np.uint64(_SM_C[1])
        z = (z ^ (z >> np.uint64(27))) * np.uint64(_SM_C[2])
        return z ^ (z >> np.uint64(31))


def _mix_torch(x):
    import torch
    def srl(v, k):
        return (v >> k) & ((1 << (64 - k)) - 1)
    z = x + _s64(_SM_C[0])
    z = (z ^ srl(z, 30)) * _s64(_SM_C[1])
    z = (z ^ srl(z, 27)) * _s64(_SM_C[2])
    return z ^ srl(z, 31)


def _h31_np(seed, j):
    return (_mix_np(_mix_np(np.asarray(j, np.uint64)) ^ np.uint64(seed)) >> np.uint64(33)).astype(np.int64)


def _h31_torch(seed, j):
    z = _mix_torch(_mix_torch(j) ^ int(seed))
    return (z >> 33) & 0x7FFFFFFF


def wide_row_ptr(m, max_len, seed, evil=()) -> np.ndarray:
    """int64 row_ptr[m+1]: row r has h(seed, r) % (max_len+1) non-zeros, except the
    (row, length) pairs in ``evil``."""
    rl = _h31_np(seed, np.arange(m, dtype=np.uint64)) % (max_len + 1)
    for r, ln in evil:
        rl[r] = ln
    rp = np.zeros(m + 1, np.int64)
    np.cumsum(rl, out=rp[1:])
    return rp


def wide_cols_vals_host(j, n, seed):
    """Columns (int32, uniform in [0, n)) and integer values {1,2,3} (fp32) of the
    global non-zeros j (numpy int64 array)."""
    j = np.asarray(j, np.int64)
    col = (_h31_np(seed + 1, j.astype(np.uint64)) % n).astype(np.int32)
    val = (1 + _h31_np(seed + 2, j.astype(np.uint64)) % 3).astype(np.float32)
    return col, val


def wide_cols_vals_device(nnz, n, seed, device="cuda", chunk=1 << 27):
    """The same arrays as wide_cols_vals_host over j = 0..nnz-1, built on the device."""
    import torch
    col = torch.empty(nnz, dtype=torch.int32, device=device)
    val = torch.empty(nnz, dtype=torch.float32, device=device)
    for j0 in range(0, nnz, chunk):
        j = torch.arange(j0, min(nnz, j0 + chunk), dtype=torch.int64, device=device)
        col[j0:j0 + j.numel()] = (_h31_torch(seed + 1, j) % n).to(torch.int32)
        val[j0:j0 + j.numel()] = (1 + _h31_torch(seed + 2, j) % 3).to(torch.float32)
        del j
    return col, val
