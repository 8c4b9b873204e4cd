"""NEXT-3 measurement: tcgen05 combination B = X*W (mps_xw_bf16) vs cuBLAS (torch.matmul,
bf16 in/out) on GCN-shaped problems.  HBM-bound: bytes = 2*n*F (X) + 2*n*N (B) + 2*F*N."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import paper_conf_ispass_shangndk23_b200 as M

PEAK = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                   "MEASURED_PEAKS.json")))["hbm_gbs"] \
    if os.path.exists("MEASURED_PEAKS.json") else 6650.0


def t(fn, reps=20):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return float(np.median(ts))


for (name, n, F, N) in [("reddit", 232965, 602, 64), ("reddit-k256", 232965, 602, 256),
                        ("products", 2449029, 100, 128), ("pubmed", 19717, 500, 16),
                        ("big-F", 1000000, 256, 256)]:
    ldx = (F + 7) // 8 * 8
    X = torch.randn(n, ldx, device="cuda").to(torch.bfloat16)[:, :F]
    W = (torch.randn(F, N, device="cuda") / F ** 0.5).to(torch.bfloat16)
    Wt = torch.zeros(N, ldx, device="cuda", dtype=torch.bfloat16)
    Wt[:, :F] = W.t()
    Wt = Wt[:, :F]
    B = torch.empty(n, N, device="cuda", dtype=torch.bfloat16)
    ours = t(lambda: M.xw_bf16(X, Wt, out=B))
    Xc = X.contiguous()
    cub = t(lambda: torch.matmul(Xc, W))
    byt = 2 * n * F + 2 * n * N + 2 * F * N
    err = (M.xw_bf16(X, Wt).float() - torch.matmul(Xc, W).float()).abs().max().item()
    print(json.dumps({"case": name, "n": n, "F": F, "N": N, "tcgen05_ms": ours, "cublas_ms": cub,
                      "tcgen05_GBps": byt / ours / 1e6, "cublas_GBps": byt / cub / 1e6,
                      "tcgen05_frac_hbm": byt / ours / 1e6 / PEAK, "max_abs_diff_vs_cublas": err,
                      "tflops": 2 * n * F * N / ours / 1e9}))
