"""NEXT-2 measurement: 2-layer GCN inference time, offline vs online merge-path schedule.

The paper reports an online-scheduling overhead of ~2% geomean, 10% on Cora and <1% on
com-Amazon (Fig. 8, RTX 6000).  Here: X (n x F) fp32, W1 F x H, W2 H x C,
out = A*(relu(A*(X*W1))*W2); CUDA events; optionally captured in CUDA graphs."""
import json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import graphgen as G
import paper_conf_ispass_shangndk23_b200 as M


def time_it(fn, steps=20, warmup=5):
    for _ in range(warmup):
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(steps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))


def main():
    F, H, C = 128, 64, 16
    res = []
    for wl in sys.argv[1:] or ["cora", "pubmed", "rmat", "reddit", "products"]:
        g = G.workload(wl)
        A = M.CSR.from_numpy(g.row_ptr, g.col_idx, g.val, g.n)
        gen = torch.Generator(device="cpu").manual_seed(0)
        X = torch.randn(g.n, F, generator=gen).cuda()
        W1 = (torch.randn(F, H, generator=gen) / F ** 0.5).cuda()
        W2 = (torch.randn(H, C, generator=gen) / H ** 0.5).cuda()
        row = {"workload": wl, "n": g.m, "nnz": g.nnz, "F": F, "H": H, "C": C}
        # default GCN2: tcgen05 combination (bf16 B) where it applies; online on a small
        # graph = the one-launch small-graph path per aggregation
        for mode in ("offline", "online", "offline_cublas", "online_cublas"):
            net = M.GCN2(A, W1, W2, online=mode.startswith("online"),
                         combination="cublas" if "cublas" in mode else "auto")
            row[mode + "_fused_online"] = bool(net.fused_online)
            row[mode + "_ms"] = time_it(lambda: net(X))
            g_ = torch.cuda.CUDAGraph()
            net(X); torch.cuda.synchronize()
            with torch.cuda.graph(g_):
                net(X)
            row[mode + "_graph_ms"] = time_it(g_.replay)
        row["online_overhead_pct"] = 100 * (row["online_ms"] / row["offline_ms"] - 1)
        row["online_overhead_graph_pct"] = 100 * (row["online_graph_ms"] / row["offline_graph_ms"] - 1)
        row["online_overhead_cublas_graph_pct"] = 100 * (row["online_cublas_graph_ms"] /
                                                         row["offline_cublas_graph_ms"] - 1)
        print(json.dumps(row), flush=True)
        res.append(row)
    ratio = [r["online_graph_ms"] / r["offline_graph_ms"] for r in res]
    print(json.dumps({"geomean_online_over_offline_graph": float(np.exp(np.mean(np.log(ratio))))}))


if __name__ == "__main__":
    main()
