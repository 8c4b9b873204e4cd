"""Torch-facing helpers over the C ABI (include/mpspmm.h).

PyTorch supplies device memory and the current stream; every step of the path runs in
libmpspmm.so.  Names follow the paper: A (CSR adjacency), B (= XW),
merge-path cost ``items_per_part``, thread floor ``min_parts``,
offline schedule.
"""
from __future__ import annotations

import ctypes
from dataclasses import dataclass

import numpy as np
import torch

from . import _lib as L

FIXUP = {"auto": L.MPS_FIXUP_AUTO, "atomic": L.MPS_FIXUP_ATOMIC, "carry": L.MPS_FIXUP_CARRY}


def _p(t):
    if t is None:
        return None
    if isinstance(t, np.ndarray):
        return ctypes.c_void_p(t.ctypes.data) if t.size else None
    return ctypes.c_void_p(t.data_ptr()) if t.numel() else None


def _stream(stream=None):
    s = torch.cuda.current_stream() if stream is None else stream
    return ctypes.c_void_p(s.cuda_stream)


def _dtype_code(B):
    if B.dtype == torch.float32:
        return L.MPS_DT_F32
    if B.dtype == torch.bfloat16:
        return L.MPS_DT_BF16
    raise TypeError("B must be float32 or bfloat16, got %s" % B.dtype)


def _fix(f):
    return FIXUP[f] if isinstance(f, str) else int(f)


class CSR:
    """A (m x n) in CSR on one device: row_ptr[m+1], int32 col_idx[nnz], fp32 val.

    row_ptr int32 uses the int32 entry points (m + nnz < 2^31); row_ptr int64 uses the
    NEXT-4 64-bit ones (mps_csr64: nnz up to 2^62, m and n < 2^31)."""

    def __init__(self, row_ptr, col_idx, val, n_cols):
        self.row_ptr, self.col_idx, self.val = row_ptr, col_idx, val
        self.m = int(row_ptr.numel()) - 1
        self.n = int(n_cols)
        self.nnz = int(col_idx.numel())
        assert row_ptr.dtype in (torch.int32, torch.int64) and col_idx.dtype == torch.int32
        assert val.dtype == torch.float32 and val.numel() == self.nnz
        self.wide = row_ptr.dtype == torch.int64

    @classmethod
    def from_numpy(cls, row_ptr, col_idx, val, n_cols, device="cuda"):
        t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).to(device)
        return cls(t(row_ptr), t(col_idx), t(val), n_cols)

    @property
    def device(self):
        return self.row_ptr.device

    def struct(self):
        cls = L.mps_csr64 if self.wide else L.mps_csr
        return cls(self.m, self.n, self.nnz, _p(self.row_ptr), _p(self.col_idx), _p(self.val))


def mps_csr_host(row_ptr, col_idx, val, n_cols) -> L.mps_csr:
    """An mps_csr holding HOST pointers (numpy arrays or pinned CPU tensors)."""
    m = (row_ptr.shape[0] if isinstance(row_ptr, np.ndarray) else row_ptr.numel()) - 1
    nnz = col_idx.shape[0] if isinstance(col_idx, np.ndarray) else col_idx.numel()
    return L.mps_csr(m, n_cols, nnz, _p(row_ptr), _p(col_idx), _p(val))


def plan(m, nnz, K, b_dtype=L.MPS_DT_F32, items_per_part=0, min_parts=0, wide=False):
    """a1: (P, L) = merge-path thread count and items per thread (Alg. 1 l.2-3).
    wide=True: mps_plan64 (no 2^31 limit on m + nnz)."""
    P, Lp = ctypes.c_int64(), ctypes.c_int64()
    f = L.mps_plan64 if wide else L.mps_plan
    f(m, nnz, K, b_dtype, items_per_part, min_parts, ctypes.byref(P), ctypes.byref(Lp))
    return P.value, Lp.value


def partition(A: CSR, num_parts, items_per_part, diag_begin=0, diag_end=None, stream=None):
    """a2: coordinates (x_p, y_p), p = 0..P, of the merge-path diagonals (Alg. 1 l.4-7)."""
    diag_end = A.m + A.nnz if diag_end is None else diag_end
    cx = _keep(torch.empty(num_parts + 1, dtype=torch.int32, device=A.device), stream)
    cy = _keep(torch.empty(num_parts + 1, dtype=A.row_ptr.dtype, device=A.device), stream)
    f = L.mps_partition64 if A.wide else L.mps_partition
    f(_p(A.row_ptr), A.m, A.nnz, diag_begin, diag_end, num_parts, items_per_part,
      _p(cx), _p(cy), _stream(stream))
    return cx, cy


@dataclass
class Schedule:
    """An offline merge-path schedule: computed once per graph, reused."""
    num_parts: int
    items_per_part: int
    coord_x: torch.Tensor
    coord_y: torch.Tensor

    @classmethod
    def build(cls, A: CSR, K, b_dtype=torch.float32, items_per_part=0, min_parts=0, stream=None):
        dt = L.MPS_DT_BF16 if b_dtype == torch.bfloat16 else L.MPS_DT_F32
        P, Lp = plan(A.m, A.nnz, K, dt, items_per_part, min_parts, wide=A.wide)
        cx, cy = partition(A, P, Lp, stream=stream)
        return cls(P, Lp, cx, cy)


def _ws(nbytes, device, stream=None):
    """Workspace for one call.  Allocated on the current stream; when the call runs on
    another ``stream`` the allocation is recorded there, so the caching allocator does
    not hand the memory out again before that stream's kernels are done with it."""
    t = torch.empty(max(int(nbytes), 1), dtype=torch.uint8, device=device)
    return _keep(t, stream)


def _keep(t, stream):
    if stream is not None and t is not None and stream != torch.cuda.current_stream(t.device):
        t.record_stream(stream)
    return t


EPILOGUE = {"none": L.MPS_EPI_NONE, "relu": L.MPS_EPI_RELU}


def spmm(A: CSR, B: torch.Tensor, schedule: Schedule | None = None, fixup="auto",
         items_per_part=0, min_parts=0, out: torch.Tensor | None = None, stream=None,
         epilogue="none"):
    """C = A * B (row-wise product) by MergePath-SpMM.

    With ``schedule`` the offline path (mps_spmm) runs; otherwise the online path
    (mps_spmm_online: plan + partition + SpMM; with the default fixup "auto" small graphs
    take the one-launch small-graph path).  B: (n, K) float32/bfloat16 on A's device,
    rows may be padded (B.stride(0) = ldb >= K).  Returns C (m, K) float32."""
    assert B.dim() == 2 and B.stride(1) == 1 and B.device == A.device
    K = B.shape[1]
    dt = _dtype_code(B)
    C = torch.empty((A.m, K), dtype=torch.float32, device=A.device) if out is None \
        else out
    if out is None:
        _keep(C, stream)
    assert C.stride(1) == 1 and C.shape == (A.m, K)
    a = A.struct()
    nb = ctypes.c_size_t()
    st = _stream(stream)
    if A.wide:      # NEXT-4: 64-bit non-zero indices
        if schedule is not None:
            L.mps_spmm64_workspace_bytes(ctypes.byref(a), K, dt, schedule.num_parts,
                                         _fix(fixup), ctypes.byref(nb))
            ws = _ws(nb.value, A.device, stream)
            L.mps_spmm64(ctypes.byref(a), _p(B), dt, B.stride(0), K, _p(C), C.stride(0),
                         _p(schedule.coord_x), _p(schedule.coord_y), schedule.num_parts,
                         _fix(fixup), EPILOGUE[epilogue], _p(ws), nb.value, st)
        else:
            L.mps_spmm64_online_workspace_bytes(ctypes.byref(a), K, dt, items_per_part,
                                                min_parts, _fix(fixup), ctypes.byref(nb))
            ws = _ws(nb.value, A.device, stream)
            L.mps_spmm64_online(ctypes.byref(a), _p(B), dt, B.stride(0), K, _p(C), C.stride(0),
                                items_per_part, min_parts, _fix(fixup), EPILOGUE[epilogue],
                                _p(ws), nb.value, st)
    elif schedule is not None:
        L.mps_spmm_workspace_bytes(ctypes.byref(a), K, dt, schedule.num_parts, _fix(fixup),
                                   ctypes.byref(nb))
        ws = _ws(nb.value, A.device, stream)
        L.mps_spmm_ex(ctypes.byref(a), _p(B), dt, B.stride(0), K, _p(C), C.stride(0),
                      _p(schedule.coord_x), _p(schedule.coord_y), schedule.num_parts,
                      _fix(fixup), EPILOGUE[epilogue], None, _p(ws), nb.value, st)
    else:
        L.mps_spmm_online_workspace_bytes(ctypes.byref(a), K, dt, items_per_part, min_parts,
                                          _fix(fixup), ctypes.byref(nb))
        ws = _ws(nb.value, A.device, stream)
        L.mps_spmm_online_ex(ctypes.byref(a), _p(B), dt, B.stride(0), K, _p(C), C.stride(0),
                             items_per_part, min_parts, _fix(fixup), EPILOGUE[epilogue],
                             _p(ws), nb.value, st)
    return C


class CapturedSpMM:
    """The online path (mps_spmm_online: partition + zeroing + segment kernel, or the
    one-launch small-graph path) captured once in a CUDA graph for fixed A, B and C
    buffers, then replayed.  Replay removes
    the per-call host launch overhead that dominates small graphs (Cora, Pubmed), and
    keeps the paper's online setting -- the schedule is recomputed on every call
    (P:151).  Update B / A values in place between replays."""

    def __init__(self, A: CSR, B: torch.Tensor, out: torch.Tensor | None = None,
                 fixup="auto", items_per_part=0, min_parts=0):
        self.A, self.B = A, B
        self.K = B.shape[1]
        self.C = torch.empty((A.m, self.K), dtype=torch.float32, device=A.device) \
            if out is None else out
        dt = _dtype_code(B)
        self.a = A.struct()
        nb = ctypes.c_size_t()
        L.mps_spmm_online_workspace_bytes(ctypes.byref(self.a), self.K, dt, items_per_part,
                                          min_parts, _fix(fixup), ctypes.byref(nb))
        self.ws = _ws(nb.value, A.device)
        args = (dt, B.stride(0), self.K, _p(self.C), self.C.stride(0), items_per_part,
                min_parts, _fix(fixup), _p(self.ws), nb.value)

        def launch():
            L.mps_spmm_online(ctypes.byref(self.a), _p(self.B), *args, _stream())
        launch()                      # first call outside capture (occupancy queries)
        torch.cuda.synchronize(A.device)
        self.graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(self.graph):
            launch()

    def __call__(self):
        self.graph.replay()
        return self.C


def xw_bf16(X: torch.Tensor, Wt: torch.Tensor, out: torch.Tensor | None = None, stream=None):
    """NEXT-3 combination B = X @ W on tcgen05 tensor cores (mps_xw_bf16).

    X: (n, F) bf16 with row stride % 8 == 0; Wt: (N, F) bf16 = W transposed; returns
    B (n, N) bf16, the row-major layout the SpMM gathers."""
    assert X.dtype == torch.bfloat16 and Wt.dtype == torch.bfloat16
    assert X.stride(1) == 1 and Wt.stride(1) == 1 and X.shape[1] == Wt.shape[1]
    n, F = X.shape

    def tma_ready(t):
        # TMA wants 16-B aligned rows: row stride % 8 bf16 and a 16-B aligned base
        if t.stride(0) % 8 == 0 and t.data_ptr() % 16 == 0:
            return t
        buf = torch.zeros((t.shape[0], -(-t.shape[1] // 8) * 8), dtype=t.dtype, device=t.device)
        buf[:, : t.shape[1]] = t
        if stream is not None:       # the staging copy must be complete before `stream` reads it
            stream.wait_stream(torch.cuda.current_stream(t.device))
        return _keep(buf, stream)[:, : t.shape[1]]
    X, Wt = tma_ready(X), tma_ready(Wt)
    N = Wt.shape[0]
    B = _keep(torch.empty((n, N), dtype=torch.bfloat16, device=X.device), stream) \
        if out is None else out
    L.mps_xw_bf16(_p(X), n, F, X.stride(0), _p(Wt), N, Wt.stride(0), _p(B), B.stride(0),
                  _stream(stream))
    return B


def spmm_host(row_ptr, col_idx, val, n_cols, B_host, C_host=None, items_per_part=0,
              min_parts=0, fixup="atomic", device="cuda", stream=None, workspace=None):
    """End to end from HOST buffers (mps_spmm_host): H2D of A and B, online SpMM, D2H
    of C, enqueued on the stream; synchronises before returning C_host."""
    K = B_host.shape[1]
    dt = L.MPS_DT_BF16 if B_host.dtype == torch.bfloat16 else L.MPS_DT_F32
    m = row_ptr.numel() - 1
    if C_host is None:
        C_host = torch.empty((m, K), dtype=torch.float32, pin_memory=True)
    a = mps_csr_host(row_ptr, col_idx, val, n_cols)
    nb = ctypes.c_size_t()
    L.mps_spmm_host_workspace_bytes(ctypes.byref(a), K, dt, B_host.stride(0), C_host.stride(0),
                                    items_per_part, min_parts, _fix(fixup), ctypes.byref(nb))
    ws = workspace if workspace is not None and workspace.numel() >= nb.value else \
        _ws(nb.value, device)
    s = torch.cuda.current_stream() if stream is None else stream
    L.mps_spmm_host(ctypes.byref(a), _p(B_host), dt, B_host.stride(0), K, _p(C_host),
                    C_host.stride(0), items_per_part, min_parts, _fix(fixup), _p(ws),
                    ws.numel(), _stream(s))
    s.synchronize()
    return C_host


def spmm_host_dense(A: CSR, B_host: torch.Tensor, C_host=None, items_per_part=0, min_parts=0,
                    fixup="atomic", stream=None, workspace=None):
    """End to end with the graph resident on A's device and B / C on the host
    (mps_spmm_host_dense: H2D of B, online SpMM, D2H of C); synchronises, returns C_host."""
    K = B_host.shape[1]
    dt = _dtype_code(B_host)
    if C_host is None:
        C_host = torch.empty((A.m, K), dtype=torch.float32, pin_memory=True)
    a = A.struct()
    nb = ctypes.c_size_t()
    L.mps_spmm_host_dense_workspace_bytes(ctypes.byref(a), K, dt, B_host.stride(0),
                                          C_host.stride(0), items_per_part, min_parts,
                                          _fix(fixup), ctypes.byref(nb))
    ws = workspace if workspace is not None and workspace.numel() >= nb.value else \
        _ws(nb.value, A.device)
    s = torch.cuda.current_stream() if stream is None else stream
    L.mps_spmm_host_dense(ctypes.byref(a), _p(B_host), dt, B_host.stride(0), K, _p(C_host),
                          C_host.stride(0), items_per_part, min_parts, _fix(fixup), _p(ws),
                          ws.numel(), _stream(s))
    s.synchronize()
    return C_host


def host_workspace_bytes(row_ptr, col_idx, val, n_cols, B_host, C_host, items_per_part=0,
                         min_parts=0, fixup="atomic"):
    K = B_host.shape[1]
    dt = L.MPS_DT_BF16 if B_host.dtype == torch.bfloat16 else L.MPS_DT_F32
    a = mps_csr_host(row_ptr, col_idx, val, n_cols)
    nb = ctypes.c_size_t()
    L.mps_spmm_host_workspace_bytes(ctypes.byref(a), K, dt, B_host.stride(0), C_host.stride(0),
                                    items_per_part, min_parts, _fix(fixup), ctypes.byref(nb))
    return nb.value


def write_stats(A: CSR, schedule: Schedule, stream=None):
    """Fig. 5 statistic: (#atomic row updates, #regular row stores) under Alg. 2."""
    cnt = _keep(torch.empty(2, dtype=torch.int64, device=A.device), stream)
    a = A.struct()
    (L.mps_write_stats64 if A.wide else L.mps_write_stats)(
        ctypes.byref(a), _p(schedule.coord_x), _p(schedule.coord_y), schedule.num_parts,
        _p(cnt), _stream(stream))
    if stream is not None:          # the counts are read on the host: wait for `stream`
        stream.synchronize()
    c = cnt.cpu()
    return int(c[0]), int(c[1])


def validate_csr(A: CSR, stream=None) -> int:
    """-1 if A's CSR content is valid, else the first offending index (synchronises)."""
    a = A.struct()
    bad = ctypes.c_int64()
    (L.mps_validate_csr64 if A.wide else L.mps_validate_csr)(ctypes.byref(a), ctypes.byref(bad), _stream(stream))
    return bad.value


class OnlineStep:
    """One online MergePath-SpMM step as the library runs it, for callers that time the
    segment kernel on its own (bench.py's path of record; the full-size parity tests run
    exactly this object).  Two forms, as ``mps_spmm_online_path`` decides:

    * partition + segments (every graph that is not small):
        a1 ``mps_plan`` (host, once) ->
        a2 + a4 zeroing: ``mps_partition_split`` (atomic; ``mps_partition`` in carry
        mode) ->
        a3 (+ a4): ``mps_spmm_segments_hot`` (dynamic segment claims from counters in the
        workspace, programmatic dependent launch behind the partition kernel);
    * small-graph fused (``MPS_PATH_SMALL_FUSED``, fixup ``auto``/``carry``): one
      ``mps_spmm_online_ex`` call -- one kernel computes the schedule and walks it, the
      carry reduction settles the cut rows.

    ``mps_spmm_online`` issues the same kernels in one call.  Buffers (workspace with the
    coordinates, C, optional hot-row bitmap) are allocated once and reused by every call,
    so a call can be captured in a CUDA graph.  ``events``: (ev_after_partition,
    ev_after_segments) recorded on the launching stream (the fused path records the first
    one before its launch).  ``cx`` / ``cy``: the schedule's coordinates after a call."""

    def __init__(self, A: CSR, K: int, b_dtype=torch.float32, fixup="atomic",
                 items_per_part=0, min_parts=0, hot="auto", out: torch.Tensor | None = None):
        assert not A.wide, "OnlineStep: int32 indices (mps_csr)"
        self.A, self.K, self.fixup = A, K, _fix(fixup)
        self.ipp, self.minp = items_per_part, min_parts
        self.dt = L.MPS_DT_BF16 if b_dtype == torch.bfloat16 else L.MPS_DT_F32
        self.a = A.struct()
        self.P, self.L = plan(A.m, A.nnz, K, self.dt, items_per_part, min_parts)
        dev = A.device
        self.C = torch.empty((A.m, K), dtype=torch.float32, device=dev) if out is None else out
        assert self.C.stride(1) == 1 and self.C.shape == (A.m, K)
        # the online workspace: [coord_x][coord_y][claim counters][carry records][...]
        nb = ctypes.c_size_t()
        L.mps_spmm_online_workspace_bytes(ctypes.byref(self.a), K, self.dt, items_per_part,
                                          min_parts, self.fixup, ctypes.byref(nb))
        self.ws_bytes = nb.value
        self.ws = _ws(nb.value, dev)
        xb = -(-(self.P + 1) * 4 // 256) * 256
        self.cx = self.ws[: (self.P + 1) * 4].view(torch.int32)
        self.cy = self.ws[xb: xb + (self.P + 1) * 4].view(torch.int32)
        self._seg_ofs = 2 * xb                     # mps_spmm_segments' workspace
        hr = ctypes.c_int64(-1)
        if hot == "auto":
            L.mps_hot_budget_rows(ctypes.byref(self.a), K, self.dt, ctypes.byref(hr))
        self.hot_rows = hr.value
        self.hot_bm = None
        if self.hot_rows >= 0:
            nbh = ctypes.c_size_t()
            L.mps_hot_rows_workspace_bytes(A.n, ctypes.byref(nbh))
            self.hot_ws_bytes = nbh.value
            self.hot_ws = _ws(nbh.value, dev)
            self.hot_bm = torch.empty((A.n + 31) // 32, dtype=torch.int32, device=dev)
        self.path = None

    def resolve(self, B: torch.Tensor) -> int:
        """The library's path for this B (MPS_PATH_*): depends on B's and C's alignment."""
        path = ctypes.c_int32()
        L.mps_spmm_online_path(ctypes.byref(self.a), _p(B), self.dt, B.stride(0), self.K,
                               _p(self.C), self.C.stride(0), self.ipp, self.minp, self.fixup,
                               ctypes.byref(path))
        return path.value

    def __call__(self, B: torch.Tensor, events=None, stream=None):
        assert B.dim() == 2 and B.stride(1) == 1 and B.shape[1] == self.K
        assert _dtype_code(B) == self.dt
        if self.path is None:
            self.path = self.resolve(B)
        s = _stream(stream)           # looked up per call: CUDA-graph capture streams
        st = stream or torch.cuda.current_stream(self.A.device)
        A, a = self.A, ctypes.byref(self.a)
        if self.path == L.MPS_PATH_SMALL_FUSED:
            if events is not None:
                events[0].record(st)
            L.mps_spmm_online_ex(a, _p(B), self.dt, B.stride(0), self.K, _p(self.C),
                                 self.C.stride(0), self.ipp, self.minp, self.fixup,
                                 L.MPS_EPI_NONE, _p(self.ws), self.ws_bytes, s)
            if events is not None:
                events[1].record(st)
            return self.C
        if self.hot_bm is not None:   # hub rows of B -> L2 evict_last (recomputed per call)
            L.mps_hot_rows(a, self.hot_rows, _p(self.hot_bm), _p(self.hot_ws),
                           self.hot_ws_bytes, s)
        if self.fixup != L.MPS_FIXUP_CARRY:      # a2 + zeroing of the cut rows, one launch
            L.mps_partition_split(_p(A.row_ptr), A.m, A.nnz, self.P, self.L, _p(self.cx),
                                  _p(self.cy), _p(self.C), self.C.stride(0), self.K, s)
        else:
            L.mps_partition(_p(A.row_ptr), A.m, A.nnz, 0, A.m + A.nnz, self.P, self.L,
                            _p(self.cx), _p(self.cy), s)
        if events is not None:
            events[0].record(st)
        seg_ws = self.ws[self._seg_ofs:]
        L.mps_spmm_segments_hot(a, _p(B), self.dt, B.stride(0), self.K, _p(self.C),
                                self.C.stride(0), _p(self.cx), _p(self.cy), self.P, self.fixup,
                                _p(self.hot_bm), _p(seg_ws), self.ws_bytes - self._seg_ofs, s)
        if events is not None:
            events[1].record(st)
        return self.C

    def launches(self, l2_bytes: int) -> int:
        """Library kernels one call launches (memsets not counted)."""
        if self.path == L.MPS_PATH_SMALL_FUSED:
            return 2
        eb = 2 if self.dt == L.MPS_DT_BF16 else 4
        tile = 512 if eb == 4 else 1024
        if self.A.n * self.K * eb > 0.5 * l2_bytes:
            tile = min(tile, 256 // eb)
        tiles = -(-self.K // min(self.K, tile)) if self.K else 0
        n = 1 + tiles * (2 if self.fixup == L.MPS_FIXUP_CARRY else 1)
        if self.hot_bm is not None:
            n += 4
        return n


def write_counts(A: CSR, B: torch.Tensor, schedule: Schedule, fixup="atomic",
                 out: torch.Tensor | None = None, stream=None):
    """Fig. 5 statistic as the segment kernel writes it (mps_spmm_write_counts): runs the
    offline SpMM with the kernel's counters on.  Returns (C, (issued partial-row updates,
    elided empty partial pieces, complete-row stores)); issued + elided is Alg. 2's
    #atomic and the last one its #regular."""
    K = B.shape[1]
    dt = _dtype_code(B)
    C = _keep(torch.empty((A.m, K), dtype=torch.float32, device=A.device), stream) \
        if out is None else out
    a = A.struct()
    nb = ctypes.c_size_t()
    L.mps_spmm_workspace_bytes(ctypes.byref(a), K, dt, schedule.num_parts, _fix(fixup),
                               ctypes.byref(nb))
    ws = _ws(nb.value, A.device, stream)
    cnt = _keep(torch.empty(3, dtype=torch.int64, device=A.device), stream)
    L.mps_spmm_write_counts(ctypes.byref(a), _p(B), dt, B.stride(0), K, _p(C), C.stride(0),
                            _p(schedule.coord_x), _p(schedule.coord_y), schedule.num_parts,
                            _fix(fixup), _p(cnt), _p(ws), nb.value, _stream(stream))
    if stream is not None:
        stream.synchronize()
    c = cnt.cpu().tolist()
    return C, (int(c[0]), int(c[1]), int(c[2]))
