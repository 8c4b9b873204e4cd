"""NEXT-1: the paper's sensitivity study on B200 (sec. V, Figs. 5-7).

For the 22 Table-II-shaped graphs (graphgen TABLE2) and K in {2, 4, 8, 16, 32, 64, 128, 256}:
  * merge-path cost sweep (items per warp segment; 0 = library default) -- Fig. 6;
  * at K=16 and the default cost: the Fig. 5 write statistic (#atomic row updates vs
    #regular row stores, mps_write_stats) and a parity check against the fp64 oracle.
Timing: the offline SpMM (split-row zeroing + segment kernel) captured in a CUDA graph,
median of 20 replays -- kernel time, as the paper's nvprof numbers.

    python tools/sensitivity.py [--out gpurun_out/sensitivity.jsonl] [--graphs a,b]
"""
import argparse, ctypes, json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import graphgen as G
import oracle as O
import paper_conf_ispass_shangndk23_b200 as M
from paper_conf_ispass_shangndk23_b200 import _lib as L
from paper_conf_ispass_shangndk23_b200.api import _p, _stream

KS = tuple(int(x) for x in os.environ.get("SENS_KS", "2 4 8 16 32 64 128 256").split())
DT = 1 if os.environ.get("SENS_DTYPE", "f32") == "bf16" else 0   # B dtype code
KS_STATS = int(os.environ.get("SENS_STATS_K", "16"))   # K of the Fig. 5 statistic + parity
COSTS = tuple(int(x) for x in os.environ.get("SENS_COSTS", "0 64 128 256 512 1024 2048 4096").split())


def replay_ms(fn, reps=20):
    fn()
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        fn()
    for _ in range(3):
        g.replay()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); g.replay(); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return float(np.median(ts))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default="gpurun_out/sensitivity.jsonl")
    ap.add_argument("--graphs", default="")
    args = ap.parse_args()
    names = [t[0] for t in G.TABLE2]
    if args.graphs:
        names = args.graphs.split(",")
    out = open(args.out, "w")
    for nm in names:
        ty = [t for t in G.TABLE2 if t[0] == nm][0][1]
        g = G.workload("t2-" + nm)
        A = M.CSR.from_numpy(g.row_ptr, g.col_idx, g.val, g.n)
        a = A.struct()
        s = _stream()
        for K in KS:
            B = torch.from_numpy(G.features(g.n, K, seed=11)).cuda()
            if DT:
                B = B.to(torch.bfloat16)
            C = torch.empty((g.m, K), device="cuda")
            for cost in COSTS:
                P, Lp = M.plan(g.m, g.nnz, K, DT, cost, 0)
                cx = torch.empty(P + 1, dtype=torch.int32, device="cuda")
                cy = torch.empty_like(cx)
                L.mps_partition(_p(A.row_ptr), g.m, g.nnz, 0, g.m + g.nnz, P, Lp, _p(cx), _p(cy), s)
                nb = ctypes.c_size_t()
                L.mps_spmm_workspace_bytes(ctypes.byref(a), K, DT, P, 1, ctypes.byref(nb))
                ws = torch.zeros(max(nb.value, 1), dtype=torch.uint8, device="cuda")

                def run():
                    L.mps_spmm(ctypes.byref(a), _p(B), DT, K, K, _p(C), K, _p(cx), _p(cy), P, 1,
                               _p(ws), nb.value, _stream())
                ms = replay_ms(run)
                row = {"graph": nm, "type": ty, "n": g.m, "nnz": g.nnz, "K": K, "cost": cost,
                       "P": P, "L": Lp, "ms": ms, "gflops": 2.0 * g.nnz * K / ms / 1e6}
                if K == KS_STATS and cost == 0:
                    cnt = torch.empty(2, dtype=torch.int64, device="cuda")
                    L.mps_write_stats(ctypes.byref(a), _p(cx), _p(cy), P, _p(cnt), s)
                    c = cnt.cpu().tolist()
                    row["writes_atomic"], row["writes_regular"] = int(c[0]), int(c[1])
                    # the same statistic counted inside the segment kernel (what it wrote)
                    sch = M.Schedule(P, Lp, cx, cy)
                    _, (iss, eli, reg) = M.write_counts(A, B, sch)
                    row["kernel_writes"] = {"atomic_issued": iss, "atomic_elided_empty": eli,
                                            "regular": reg}
                    row["kernel_counts_match"] = (iss + eli, reg) == (int(c[0]), int(c[1]))
                    run()
                    torch.cuda.synchronize()
                    ref, bnd = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B.float().cpu().numpy())
                    row["parity_ok"] = bool(O.check(C.cpu().numpy(), ref, bnd)["ok"])
                out.write(json.dumps(row) + "\n")
                out.flush()
        print(nm, "done", flush=True)
    out.close()


if __name__ == "__main__":
    main()
