"""Segment-kernel microbenchmark: back-to-back launches vs. the bench's step order."""
import ctypes, sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, numpy as np
import graphgen as G
import paper_conf_ispass_shangndk23_b200 as M
from paper_conf_ispass_shangndk23_b200 import _lib as L
from paper_conf_ispass_shangndk23_b200.api import _p, _stream

wl = sys.argv[1] if len(sys.argv) > 1 else "reddit"
K = int(sys.argv[2]) if len(sys.argv) > 2 else 64
dt = sys.argv[3] if len(sys.argv) > 3 else "f32"
g = G.workload(wl); B = torch.from_numpy(G.features(wl, K)).cuda()
if dt == "bf16":
    B = B.to(torch.bfloat16)
DT = 1 if dt == "bf16" else 0
A = M.CSR.from_numpy(g.row_ptr, g.col_idx, g.val, g.n)
a = A.struct(); s = _stream()
P, Lp = M.plan(g.m, g.nnz, K, DT)
cx = torch.empty(P + 1, dtype=torch.int32, device="cuda"); cy = torch.empty_like(cx)
C = torch.empty(g.m, K, device="cuda")
L.mps_partition(_p(A.row_ptr), g.m, g.nnz, 0, g.m + g.nnz, P, Lp, _p(cx), _p(cy), s)
nb = ctypes.c_size_t()
L.mps_spmm_workspace_bytes(ctypes.byref(a), K, DT, P, 1, ctypes.byref(nb))
ws = torch.zeros(max(nb.value, 1), dtype=torch.uint8, device="cuda")
def seg():
    L.mps_spmm_segments(ctypes.byref(a), _p(B), DT, K, K, _p(C), K, _p(cx), _p(cy), P, 1, _p(ws), nb.value, s)
def zero():
    L.mps_zero_split_rows(ctypes.byref(a), _p(cx), _p(cy), P, _p(C), K, K, s)
def timeit(fn, pre=None, n=6):
    out = []
    for _ in range(n):
        if pre: pre()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize(); out.append(e0.elapsed_time(e1))
    return [round(x, 3) for x in out]
zero(); seg(); torch.cuda.synchronize()
res = {"back_to_back": timeit(seg), "after_zero": timeit(seg, pre=zero)}
flush = torch.empty(64 * 1024 * 1024, device="cuda")
res["after_flush_zero"] = timeit(seg, pre=lambda: (flush.zero_(), zero()))
torch.cuda.synchronize()
print(json.dumps(res))
