"""NEXT-4 measurement: the 64-bit-index path (mps_csr64) on a graph past 2^31 non-zeros,
and the int32 vs int64 cost of the same kernel on the BASELINE graphs.

Usage (GPU box): python tools/wide_bench.py [--out gpurun_out/wide.jsonl]
Each line: workload, index width, B dtype, K, ms per online step (median of timed steps,
L2 flushed before each), GFLOP/s (2 nnz K / t) and the segment kernel's algorithmic
GB/s (8 nnz + idx (m+1) + b_elt nnz K + 4 m K per launch).
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import graphgen as G
import paper_conf_ispass_shangndk23_b200 as M


def time_step(A, B, steps=10, warmup=3):
    flush = torch.empty(2 * 128 * 1024 * 1024 // 4, device="cuda")
    C = torch.empty(A.m, B.shape[1], device="cuda")
    ts = []
    for i in range(warmup + steps):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        M.spmm(A, B, out=C)
        e1.record()
        torch.cuda.synchronize()
        if i >= warmup:
            ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))


def line(name, A, B, t, out):
    K = B.shape[1]
    eb = B.element_size()
    idx = A.row_ptr.element_size()
    alg = 8 * A.nnz + idx * (A.m + 1) + eb * A.nnz * K + 4 * A.m * K
    rec = {"workload": name, "index": "int64" if A.wide else "int32",
           "b_dtype": "bf16" if eb == 2 else "f32", "K": K, "m": A.m, "nnz": A.nnz,
           "ms": round(t, 4), "gflops": round(2 * A.nnz * K / t / 1e6, 1),
           "alg_gbs": round(alg / t / 1e6, 1)}
    print(json.dumps(rec), flush=True)
    out.write(json.dumps(rec) + "\n")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default="gpurun_out/wide_bench.jsonl")
    ap.add_argument("--skip-wide", action="store_true")
    a = ap.parse_args()
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out, "w") as out:
        for wl, K in (("reddit", 64), ("products", 128), ("rmat", 64)):
            g = G.workload(wl)
            B = torch.from_numpy(G.features(wl, K)).cuda()
            for wide in (False, True):
                rp = g.row_ptr.astype(np.int64) if wide else g.row_ptr
                A = M.CSR.from_numpy(rp, g.col_idx, g.val, g.n)
                line(wl, A, B, time_step(A, B), out)
            del A, B
            torch.cuda.empty_cache()
        if a.skip_wide:
            return
        # past 2^31 non-zeros: 2.62 M rows x ~1025 non-zeros (+3 rows of 10^6), 1 M columns
        m, n, seed = 2_621_440, 1 << 20, 41
        rp = G.wide_row_ptr(m, 2048, seed, [(0, 10 ** 6), (m // 2 + 3, 10 ** 6), (m - 1, 10 ** 6)])
        nnz = int(rp[-1])
        col, val = G.wide_cols_vals_device(nnz, n, seed)
        A = M.CSR(torch.from_numpy(rp).cuda(), col, val, n)
        for K in (16, 64):
            B = torch.from_numpy(G.dense_uniform(n, K, seed)).cuda()
            line("wide-2.7e9", A, B, time_step(A, B, steps=5), out)
            line("wide-2.7e9", A, B.to(torch.bfloat16), time_step(A, B.to(torch.bfloat16), steps=5),
                 out)


if __name__ == "__main__":
    main()
