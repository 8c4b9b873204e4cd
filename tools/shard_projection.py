"""Per-GPU work of the merge-path sharder at G = 1, 2, 4, 8, measured on ONE B200.

For each G and each rank g < G, the rank's ShardedSpMM (full row_ptr, its col/val slice
[Y_g, Y_{g+1}), the replicated B) runs its local step -- partition of its diagonals,
segment kernel(s) over all column tiles, tail row into the tail buffer -- alone on the
GPU, L2 flushed before every launch, CUDA events, median of `reps`.  t_G = max over
ranks; S_G = t_1 / t_G.  This is a projection: on G GPUs each rank runs exactly this
launch sequence on its own GPU with its own L2 and HBM, plus the tail exchange (the fused
peer-memory epilogue or one all-gather of G*K floats, ~10-30 us), which is not included.
Usage: python tools/shard_projection.py [workload K [reps]]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import graphgen as G
import paper_conf_ispass_shangndk23_b200 as M

wl = sys.argv[1] if len(sys.argv) > 1 else "products"
K = int(sys.argv[2]) if len(sys.argv) > 2 else 128
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 7
g = G.workload(wl)
Bd = torch.from_numpy(G.features(wl, K)).cuda()
l2 = torch.cuda.get_device_properties(0).L2_cache_size
flush = torch.empty(2 * l2 // 4, device="cuda")
flush_clean = torch.zeros_like(flush)
sink = torch.empty(1, device="cuda")
res = {"workload": "%s-k%d" % (wl, K), "n": g.m, "nnz": g.nnz, "per_G": {}}
t1 = None
ipp = int(os.environ.get("IPP", "0"))
for world in [int(x) for x in os.environ.get("GS", "1 2 4 8").split()]:
    per_rank = []
    for rank in range(world):
        sh = M.ShardedSpMM(g.row_ptr, g.col_idx, g.val, g.n, K, rank, world, "cuda",
                           items_per_part=ipp)
        sh.local(Bd)
        torch.cuda.synchronize()
        ts = []
        for _ in range(reps):
            flush.zero_()                 # bench.py's flush: write 2x L2, read 2x L2
            torch.sum(flush_clean, dim=0, out=sink[0])
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            sh.local(Bd)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        per_rank.append(float(np.median(ts)))
        del sh
        torch.cuda.empty_cache()
    tg = max(per_rank)
    t1 = tg if t1 is None else t1
    res["per_G"][world] = {"t_ms_max_rank": round(tg, 4),
                           "t_ms_per_rank": [round(x, 4) for x in per_rank],
                           "projected_speedup": round(t1 / tg, 2),
                           "gflops_projected": round(2.0 * g.nnz * K / (tg * 1e-3) / 1e9, 1)}
    print(json.dumps({world: res["per_G"][world]}), flush=True)
print(json.dumps(res))
