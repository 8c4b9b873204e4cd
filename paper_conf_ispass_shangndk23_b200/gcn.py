"""NEXT-2: two-layer GCN inference on MergePath-SpMM.

    out = A · ( relu( A · (X · W1) ) · W2 )           (A·(X·W) order P:282)

The combination X·W runs on the library's tcgen05 kernel (``mps_xw_bf16``, B in bf16
straight into the gather layout; 1.2-3.3x cuBLAS on the GCN shapes, profiles/r02) wherever
it applies (16 <= N <= 256, N % 16 == 0: ``combination="auto"``, the default), else as a
plain cuBLAS GEMM (torch.matmul, fp32 B).  The aggregation A·B is MergePath-SpMM (libmpspmm), with the
layer-1 ReLU fused into it (MPS_EPI_RELU: complete rows at the store, cut rows after
their partial sums).  ``online=True`` recomputes the merge-path
schedule on every inference (the paper's online setting) -- one partition per
inference serves both layers; ``online=False`` computes it once and reuses it for every
call (the offline default).
"""
from __future__ import annotations

import ctypes

import torch

from .api import CSR, Schedule, spmm, xw_bf16


class GCN2:
    def __init__(self, A: CSR, W1: torch.Tensor, W2: torch.Tensor, online: bool = False,
                 b_dtype=torch.float32, fixup: str = "auto", items_per_part: int = 0,
                 min_parts: int = 0, combination: str = "auto"):
        self.A, self.W1, self.W2 = A, W1, W2
        self.online, self.b_dtype, self.fixup = online, b_dtype, fixup
        # "tcgen05": X*W by the library's tensor-core kernel (mps_xw_bf16), B in bf16
        # straight into the gather layout (NEXT-3); "cublas": torch.matmul
        if combination == "auto":
            # tcgen05 where the kernel applies, except tiny graphs: on Cora (2,708 rows)
            # cuBLAS's X*W is 4 us faster per inference, from Pubmed (19,717) up tcgen05
            # wins (profiles/r02/gcn_online_offline.md)
            ok = all(16 <= w.shape[1] <= 256 and w.shape[1] % 16 == 0 for w in (W1, W2))
            combination = "tcgen05" if ok and A.m >= 8192 else "cublas"
        self.combination = combination
        if combination == "tcgen05":
            self.b_dtype = torch.bfloat16
            self.W1t = W1.t().contiguous().to(torch.bfloat16)
            self.W2t = W2.t().contiguous().to(torch.bfloat16)
        self.ipp, self.minp = items_per_part, min_parts
        self.H = torch.empty((A.m, W1.shape[1]), dtype=torch.float32, device=A.device)
        self.out = torch.empty((A.m, W2.shape[1]), dtype=torch.float32, device=A.device)
        # the default plan depends on the graph only, so one schedule serves both layers
        self.schedule = None if online else Schedule.build(A, W1.shape[1], self.b_dtype,
                                                           items_per_part, min_parts)
        # online on a small graph: each aggregation is one mps_spmm_online call on the
        # one-launch small-graph path (it computes its own schedule inside the kernel)
        self.fused_online = False
        if online and not A.wide:
            from . import _lib as L
            path = ctypes.c_int32()
            a = A.struct()
            ok = True
            for w in (W1, W2):
                L.mps_spmm_online_path(ctypes.byref(a), None,
                                       L.MPS_DT_BF16 if self.b_dtype == torch.bfloat16
                                       else L.MPS_DT_F32, w.shape[1], w.shape[1], None,
                                       w.shape[1], items_per_part, min_parts,
                                       L.MPS_FIXUP_AUTO if fixup == "auto" else
                                       (L.MPS_FIXUP_CARRY if fixup == "carry" else
                                        L.MPS_FIXUP_ATOMIC), ctypes.byref(path))
                ok = ok and path.value == L.MPS_PATH_SMALL_FUSED
            self.fused_online = ok

    def _aggregate(self, B, out, epilogue):
        if self.fused_online:
            return spmm(self.A, B.to(self.b_dtype), fixup=self.fixup, items_per_part=self.ipp,
                        min_parts=self.minp, out=out, epilogue=epilogue)
        return spmm(self.A, B.to(self.b_dtype), schedule=self.schedule, fixup=self.fixup,
                    items_per_part=self.ipp, min_parts=self.minp, out=out, epilogue=epilogue)

    def _combine(self, X, W, Wt):
        if self.combination == "tcgen05":
            return xw_bf16(X.to(torch.bfloat16), Wt)
        return X @ W

    def layer1(self, X: torch.Tensor) -> torch.Tensor:
        return self._aggregate(self._combine(X, self.W1, getattr(self, "W1t", None)), self.H,
                               "relu")

    def __call__(self, X: torch.Tensor) -> torch.Tensor:
        if self.online and not self.fused_online:
            # online setting: the schedule is recomputed for every inference --
            # once, since the default plan depends on the graph only, for both layers
            self.schedule = Schedule.build(self.A, self.W1.shape[1], self.b_dtype, self.ipp,
                                           self.minp)
        H = self.layer1(X)
        return self._aggregate(self._combine(H, self.W2, getattr(self, "W2t", None)), self.out,
                               "none")
