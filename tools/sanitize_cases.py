"""Small cases covering every segment-kernel variant, fix-up mode and edge path, for
compute-sanitizer (memcheck / racecheck / synccheck).  Exits non-zero on a mismatch."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import graphgen as G
import oracle as O
import paper_conf_ispass_shangndk23_b200 as M


def run():
    rs = np.random.RandomState(0)
    bad = 0
    for K in (1, 4, 16, 32, 64, 96, 128, 256, 520):
        for dt in (torch.float32, torch.bfloat16):
            m = int(rs.randint(50, 400))
            rl = rs.randint(0, 20, size=m).astype(np.int32)
            rl[rs.randint(m)] = 900
            g = G.random_csr(m, 300, rl, K)
            # exact-size allocations (no padding): TMA tail / remainder paths are exercised
            A = M.CSR(torch.from_numpy(g.row_ptr).cuda(), torch.from_numpy(g.col_idx).cuda(),
                      torch.from_numpy(g.val).cuda(), g.n)
            B = G.dense_int(300, K, seed=K)
            ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
            Bt = torch.from_numpy(B).cuda().to(dt)
            # "auto": the one-launch small-graph path (small.cu) + carry reduction
            for fixup in ("atomic", "carry", "auto"):
                for cost in (7, 64, 2048):
                    C = M.spmm(A, Bt, fixup=fixup, items_per_part=cost, min_parts=1)
                    torch.cuda.synchronize()
                    if not np.array_equal(C.cpu().numpy().astype(np.float64), ref):
                        print("MISMATCH", K, dt, fixup, cost)
                        bad += 1
    # dynamic segment claims (more segments than resident warps), repeated launches
    rl = rs.randint(0, 9, size=12000).astype(np.int32)
    rl[rs.rand(12000) < 0.3] = 0
    rl[777] = 5000
    g = G.random_csr(12000, 2000, rl, 77)
    A = M.CSR(torch.from_numpy(g.row_ptr).cuda(), torch.from_numpy(g.col_idx).cuda(),
              torch.from_numpy(g.val).cuda(), g.n)
    for K, dt in ((64, torch.float32), (32, torch.bfloat16)):
        B = G.dense_int(2000, K, seed=K)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        for fixup in ("atomic", "carry"):
            for _ in range(2):
                C = M.spmm(A, torch.from_numpy(B).cuda().to(dt), fixup=fixup, items_per_part=2,
                           min_parts=1)
                torch.cuda.synchronize()
                if not np.array_equal(C.cpu().numpy().astype(np.float64), ref):
                    print("MISMATCH dynamic claims", K, dt, fixup)
                    bad += 1
    # bf16 next-batch L2 prefetch forced on (dynamic claims; 4, 2 and 1 rows per
    # instruction)
    os.environ["MPS_PF"] = "1"
    for K in (64, 128, 256):
        B = G.dense_int(2000, K, seed=K + 5)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        for fixup in ("atomic", "carry"):
            C = M.spmm(A, torch.from_numpy(B).cuda().to(torch.bfloat16), fixup=fixup,
                       items_per_part=2, min_parts=1)
            torch.cuda.synchronize()
            if not np.array_equal(C.cpu().numpy().astype(np.float64), ref):
                print("MISMATCH bf16 prefetch", K, fixup)
                bad += 1
    del os.environ["MPS_PF"]
    # deep-gather instantiation forced on (fp32, 64-column tiles), static and dynamic
    os.environ["MPS_DEEP"] = "1"
    os.environ["MPS_TILE"] = "64"
    for K in (64, 128):
        B = G.dense_int(2000, K, seed=K)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        for fixup in ("atomic", "carry"):
            for cost in (2, 0):
                C = M.spmm(A, torch.from_numpy(B).cuda(), fixup=fixup, items_per_part=cost,
                           min_parts=1 if cost else 0)
                torch.cuda.synchronize()
                if not np.array_equal(C.cpu().numpy().astype(np.float64), ref):
                    print("MISMATCH deep", K, fixup, cost)
                    bad += 1
    del os.environ["MPS_DEEP"], os.environ["MPS_TILE"]
    # shard path (loopback)
    g = G.random_csr(80, 60, np.r_[np.ones(40, np.int32), [700], np.ones(39, np.int32)], 3)
    B = G.dense_int(60, 12, seed=1)
    Bt = torch.from_numpy(B).cuda()
    sh = [M.ShardedSpMM(g.row_ptr, g.col_idx, g.val, g.n, 12, r, 3, "cuda", items_per_part=9,
                        min_parts=1) for r in range(3)]
    for s in sh:
        s.local(Bt)
    tails = torch.cat([s.tail for s in sh])
    out = np.concatenate([s.settle(tails).cpu().numpy() for s in sh])
    ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
    if not np.array_equal(out.astype(np.float64), ref):
        print("MISMATCH shard")
        bad += 1
    # NEXT-4: int64 row_ptr / nnz coordinates
    for K in (4, 64, 128):
        for dt in (torch.float32, torch.bfloat16):
            m = int(rs.randint(50, 400))
            rl = rs.randint(0, 20, size=m).astype(np.int32)
            rl[rs.randint(m)] = 900
            g = G.random_csr(m, 300, rl, K + 1)
            A = M.CSR(torch.from_numpy(g.row_ptr.astype(np.int64)).cuda(),
                      torch.from_numpy(g.col_idx).cuda(), torch.from_numpy(g.val).cuda(), g.n)
            B = G.dense_int(300, K, seed=K)
            ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
            for fixup in ("atomic", "carry"):
                for cost in (7, 2048):
                    C = M.spmm(A, torch.from_numpy(B).cuda().to(dt), fixup=fixup,
                               items_per_part=cost, min_parts=1)
                    torch.cuda.synchronize()
                    if not np.array_equal(C.cpu().numpy().astype(np.float64), ref):
                        print("MISMATCH int64", K, dt, fixup, cost)
                        bad += 1
    # NEXT-3: tcgen05 combination, single destination and 3-replica loopback broadcast
    import ctypes
    from paper_conf_ispass_shangndk23_b200.api import _p, _stream
    gen = torch.Generator().manual_seed(0)
    n, F, N = 777, 72, 64
    X = torch.randint(-1, 2, (n, F), generator=gen).to(torch.bfloat16)
    W = torch.randint(-1, 2, (F, N), generator=gen).to(torch.bfloat16)
    ref = X.double() @ W.double()
    Xd, Wt = X.cuda(), W.t().contiguous().cuda()
    if not torch.equal(M.xw_bf16(Xd, Wt).double().cpu(), ref):
        print("MISMATCH xw")
        bad += 1
    reps = [torch.zeros((n, N), dtype=torch.bfloat16, device="cuda") for _ in range(3)]
    for r in range(3):
        r0, r1 = M.row_block(n, 3, r)
        arr = (ctypes.c_void_p * 3)(*[reps[(r + k) % 3].data_ptr() for k in range(3)])
        M.mps_xw_bf16_bcast(_p(Xd[r0:r1]), r1 - r0, F, F, _p(Wt), N, F, arr, 3, r0, N,
                            _stream())
    torch.cuda.synchronize()
    if not all(torch.equal(t.double().cpu(), ref) for t in reps):
        print("MISMATCH xw bcast")
        bad += 1
    # B as wide as X (N >= F): the 3-stage ring, TMA-store epilogue, partial last tile
    n, F, N = 1000, 64, 128
    X = torch.randint(-1, 2, (n, F), generator=gen).to(torch.bfloat16)
    W = torch.randint(-1, 2, (F, N), generator=gen).to(torch.bfloat16)
    if not torch.equal(M.xw_bf16(X.cuda(), W.t().contiguous().cuda()).double().cpu(),
                       X.double() @ W.double()):
        print("MISMATCH xw N >= F")
        bad += 1
    print("sanitize cases done, mismatches:", bad)
    return bad


if __name__ == "__main__":
    sys.exit(1 if run() else 0)
