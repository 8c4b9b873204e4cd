#!/usr/bin/env python
"""MergePath-SpMM benchmark (BASELINE.json metric: SpMM GFLOP/s = 2*nnz*K / t, with the
effective HBM GB/s and the HBM-roofline fraction beside it).

One step = one pass of the whole hot path of SURVEY.md sec. 8(a) on one batch:
a1 plan (host) + a2 partition + a4 split-row zeroing + a3 segment kernel (+ a4 carry
reduction) and, for N > 1 GPUs, the a6 tail all-gather + tail application.  Inputs
(A, B) are resident in HBM; L2 is flushed (a 2x-L2 write) before every timed step, and
each step is timed with CUDA events on the launching stream.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload reddit] [--K 64]
                    [--fixup atomic|carry] [--dtype f32|bf16] [--impl reference]

N > 1: launch under torchrun (one rank per GPU, NCCL); rank 0 prints the JSON line.
"""
from __future__ import annotations

import argparse
import ctypes
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "SpMM GFLOP/s (2·nnz·K) & HBM GB/s vs 8 TB/s at 1/2/4/8 B200"
# The paper's own results: ratios on other hardware, context only
PAPER_CONTEXT = {
    "hardware": "NVIDIA Quadro RTX 6000 (Turing sm_75, 72 SMs, 672 GB/s), fp32 presumed (P:159)",
    "speedups": {
        "vs GNNAdvisor, geomean over 22 Table-II graphs, K=16": "1.85x (P:230)",
        "vs GNNAdvisor-opt": "+31% (P:230)",
        "online scheduling overhead, 2-layer GCN, geomean": "~2% (P:282)",
        "online overhead Cora / com-Amazon": "10% / <1% (P:282)",
    },
    "absolute_numbers": None,
    "note": "the paper prints no absolute time or GFLOP/s; not a target (vs_baseline null)",
}
FALLBACK_HBM_GBS = 6650.0   # B200_PROFILING.md fallback, used only without MEASURED_PEAKS.json


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--workload", default="reddit")
    ap.add_argument("--K", type=int, default=0)
    ap.add_argument("--fixup", default="auto", choices=["auto", "atomic", "carry"],
                    help="a4 fix-up: auto = the library's choice (carry on the small-graph "
                         "fused path, atomic otherwise)")
    ap.add_argument("--dtype", default="f32", choices=["f32", "bf16"])
    ap.add_argument("--items-per-part", type=int, default=0)
    ap.add_argument("--min-parts", type=int, default=0)
    ap.add_argument("--impl", default="mps", choices=["mps", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--out", default="")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="N > 1 process-group backend (gloo: CPU-staged tails, for testing "
                         "several ranks on one GPU)")
    ap.add_argument("--no-cusparse", action="store_true",
                    help="skip the cuSPARSE reference point (N=1, fp32)")
    ap.add_argument("--no-l2-probe", action="store_true",
                    help="skip the live L2 read-bandwidth ceiling (roofline.units)")
    ap.add_argument("--tails", default="auto", choices=["auto", "p2p", "nccl"],
                    help="N>1 tail exchange: p2p = fused into the final kernel over peer "
                         "memory (auto: p2p if it sets up and cross-checks, else nccl)")
    ap.add_argument("--extras", action="store_true",
                    help="N>1: also time the NEXT-3 fused combination + replication and one "
                         "pipelined GCN layer (reported in b_replication, not in the step)")
    ap.add_argument("--hot", default="auto", choices=["auto", "off"],
                    help="degree-aware L2 residency of B rows (auto: when B exceeds L2/2)")
    ap.add_argument("--cuda-graph", action="store_true",
                    help="capture each step in a CUDA graph and replay it (launch-bound graphs)")
    ap.add_argument("--flush", default="write", choices=["write", "read", "none"],
                    help="L2 flush before each timed step: write (default) or read a 2x-L2 "
                         "buffer, or none")
    return ap.parse_args()


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md 6.65 TB/s)"


def alg_bytes(m, nnz, K, b_elt):
    """nnz*(4 idx + 4 val) + 4*(m+1) row_ptr + b_elt*nnz*K gathered B rows
    + 4*m*K for C."""
    return 8 * nnz + 4 * (m + 1) + b_elt * nnz * K + 4 * m * K


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index, self.proc, self.lines = index, None, []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), "--query-gpu=" + self.Q,
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 6:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[2:6]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None,
                "sm_max_mhz": float(max(mx)) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def cpu_oracle_rate(g, B, K, seconds, steps=1):
    """Time the oracle O1 (fp64, OpenMP over rows) on a bounded row sample of the same
    workload; returns (GFLOP/s, cores, sample description, seconds per step)."""
    import oracle as O
    rows_all = g.m
    deg = np.diff(g.row_ptr).astype(np.int64)
    # calibrate on a small prefix, then size the sample to `seconds`
    r0 = max(1, min(rows_all, 2000))
    t = time.perf_counter()
    O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, rows=np.arange(r0), want_bound=False)
    dt = max(time.perf_counter() - t, 1e-6)
    rate_nnz = deg[:r0].sum() / dt
    want_nnz = rate_nnz * seconds / max(steps, 1)
    cum = np.cumsum(deg)
    R = int(np.searchsorted(cum, want_nnz)) + 1
    R = max(1, min(rows_all, R))
    rows = np.arange(R, dtype=np.int64)
    times = []
    for _ in range(steps):
        t = time.perf_counter()
        O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, rows=rows, want_bound=False)
        times.append(time.perf_counter() - t)
    nnz_s = int(cum[R - 1])
    gflop = 2.0 * nnz_s * K / 1e9
    tm = float(np.median(times))
    sample = ("rows [0, %d) of %s (%d of %d nnz, %.1f%%), K=%d, fp64 oracle O1" %
              (R, g.name, nnz_s, g.nnz, 100.0 * nnz_s / max(g.nnz, 1), K))
    return gflop / tm, O.num_threads(), sample, tm


def run_reference(args):
    """--impl reference: the CPU oracle (as it stands) on a bounded sample per step."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import graphgen as G
    g = G.workload(args.workload)
    K = args.K or G.WORKLOADS[args.workload][3][0]
    B = G.features(args.workload, K)
    per_step = max(1.0, 90.0 / max(1, args.steps + args.warmup))
    rate, cores, sample, tm = cpu_oracle_rate(g, B, K, per_step * (args.steps), args.steps)
    line = {
        "metric": METRIC, "value": rate, "unit": "GFLOP/s", "impl": "reference",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": tm * 1e3, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": "%s-k%d" % (args.workload, K), "n": g.m, "nnz": g.nnz, "K": K},
        "cpu_baseline": {"value": rate, "unit": "GFLOP/s", "cores": cores, "kind": "oracle",
                         "sample": sample},
        "e2e": {"value": rate, "unit": "GFLOP/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
        "gpu_launches": 0,
    }
    print(json.dumps(line), flush=True)


def n_tile_cols(n, K, b_elt, l2):
    """Columns per tile the library runs for K (capi.cu choose_vec with aligned buffers):
    32 lanes x 16 B x 4 slots per pass, 256-B row slices when B exceeds half the L2."""
    t = 512 if b_elt == 4 else 1024
    if n * K * b_elt > 0.5 * l2:
        t = min(t, 256 // b_elt)
    return t


def n_tiles(n, K, b_elt, l2):
    return -(-K // min(K, n_tile_cols(n, K, b_elt, l2)))


# L2 read ceiling when the live probe is skipped (--no-l2-probe): the lean random-gather
# probe measured on this pool's B200s (profiles/r02/l2_probe.md)
L2_PEAK_FALLBACK_GBS = 20300.0
L2_PEAK_FALLBACK_SRC = "fallback: lean L2 gather probe measured in round 2 (profiles/r02)"


def validate_output(g, Bd, C, cx, cy, K, n_random=2000, seed=0):
    """Parity of the timed step's C (untimed, after the timed region): every row cut by
    a merge-path boundary (the rows a4 settles), random rows and the 50 longest rows
    against the fp64 oracle O1/O2 within |C - C_ref| <= 1e-5 (|A||B|) + 1e-7, every
    column sum of the whole C against w^T B (w = column sums of A, fp64; allowed error
    1e-5 |w|^T|B| + m 1e-7, the sum of the element bounds), and no NaN/Inf anywhere."""
    import torch
    import oracle as O
    t0 = time.perf_counter()
    B = Bd.float().cpu().numpy()            # bf16 B: the oracle sees the rounded values
    cxh, cyh = cx.cpu().numpy(), cy.cpu().numpy()
    inside = (cxh < g.m) & (cyh > g.row_ptr[np.minimum(cxh, g.m)])
    cut = np.unique(cxh[inside]).astype(np.int64)
    rs = np.random.RandomState(seed)
    deg = np.diff(g.row_ptr)
    rows = np.unique(np.concatenate([cut, rs.randint(0, g.m, n_random), np.argsort(deg)[-50:],
                                     [0, g.m - 1]]).astype(np.int64))
    ref, bnd = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, rows=rows)
    got = C[torch.from_numpy(rows).to(C.device)].cpu().numpy()
    r = O.check(got, ref, bnd)
    w = np.bincount(g.col_idx, weights=g.val.astype(np.float64), minlength=g.n)
    B64 = B.astype(np.float64)
    cs_ref, cs_abs = w @ B64, np.abs(w) @ np.abs(B64)
    cs = C.double().sum(0).cpu().numpy()
    cs_ok = bool(np.all(np.abs(cs - cs_ref) <= 1e-5 * cs_abs + g.m * 1e-7))
    nonfinite = int((~torch.isfinite(C)).sum())
    return {"ok": bool(r["ok"] and cs_ok and nonfinite == 0), "rows_checked": int(len(rows)),
            "cut_rows_checked": int(len(cut)), "worst_err_over_tol": r["worst_ratio"],
            "violations": r["violations"], "colsums_ok": cs_ok, "nonfinite_in_C": nonfinite,
            "tolerance": "|C - C_ref| <= 1e-5 (|A||B|) + 1e-7 (north star), fp64 oracle O1",
            "seconds": round(time.perf_counter() - t0, 2)}


def validate_output_shard(g, Bd, sh, K, rank, n_random=500, seed=0):
    """N > 1: this rank's final rows [X_g, X_{g+1}) (tails applied): its first and last
    rows, the longest and random rows against O1/O8, and the column sums of its rows."""
    import torch
    import oracle as O
    t0 = time.perf_counter()
    r0, r1 = int(sh.X[rank]), int(sh.X[rank + 1])
    if r1 <= r0:
        return {"ok": True, "rows_checked": 0, "seconds": 0.0}
    B = Bd.float().cpu().numpy()
    C = sh.C[: r1 - r0]
    rs = np.random.RandomState(seed + rank)
    deg = np.diff(g.row_ptr[r0:r1 + 1])
    loc = np.unique(np.concatenate([rs.randint(0, r1 - r0, n_random),
                                    np.argsort(deg)[-20:], [0, r1 - r0 - 1]])).astype(np.int64)
    ref, bnd = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, rows=loc + r0)
    r = O.check(C[torch.from_numpy(loc).to(C.device)].cpu().numpy(), ref, bnd)
    j0, j1 = int(g.row_ptr[r0]), int(g.row_ptr[r1])
    w = np.bincount(g.col_idx[j0:j1], weights=g.val[j0:j1].astype(np.float64), minlength=g.n)
    B64 = B.astype(np.float64)
    cs_ref, cs_abs = w @ B64, np.abs(w) @ np.abs(B64)
    cs = C.double().sum(0).cpu().numpy()
    cs_ok = bool(np.all(np.abs(cs - cs_ref) <= 1e-5 * cs_abs + (r1 - r0) * 1e-7))
    nonfinite = int((~torch.isfinite(C)).sum())
    return {"ok": bool(r["ok"] and cs_ok and nonfinite == 0), "rows_checked": int(len(loc)),
            "worst_err_over_tol": r["worst_ratio"], "colsums_ok": cs_ok,
            "nonfinite_in_C": nonfinite, "seconds": round(time.perf_counter() - t0, 2)}


# input feature width F of the combination X*W per workload (the datasets' feature sizes;
# synthetic R-MAT: 64)
FEATURES = {"cora": 1433, "pubmed": 500, "reddit": 602, "products": 100, "rmat": 64}


def xw_replication(M, g, K, rank, world, dev, stream):
    """NEXT-3 multi-GPU: produce the replicated B (bf16) from row-sharded X.
    fused: ONE kernel per rank (mps_xw_bf16_bcast) computes its row block of X*W and stores
    it into every rank's replica over NVLink (CUDA IPC peer pointers);
    unfused: the same GEMM into the local block, then NCCL all_gather_into_tensor.
    Times are CUDA events on the launching stream, max over ranks, best of 3."""
    import torch
    import torch.distributed as dist
    F = FEATURES.get(g.name.split("-")[0], 64)
    ldx = -(-F // 8) * 8
    r0, r1 = M.row_block(g.n, world, rank)
    gen = torch.Generator(device="cpu").manual_seed(1000 + rank)
    X = torch.zeros((max(r1 - r0, 1), ldx), dtype=torch.bfloat16)
    X[:, :F] = torch.randn(X.shape[0], F, generator=gen).to(torch.bfloat16)
    X = X.to(dev)[: r1 - r0, :F]
    Wt = torch.zeros((K, ldx), dtype=torch.bfloat16)
    Wt[:, :F] = (torch.randn(K, F, generator=torch.Generator().manual_seed(7)) / F ** 0.5)
    Wt = Wt.to(dev)[:, :F]
    rep = M.PeerReplicas(g.n, K, rank, world, dev)
    nccl = dist.get_backend() == "nccl"
    per = -(-g.n // world)
    full = torch.empty((per * world, K), dtype=torch.bfloat16, device=dev)
    fused, unfused = [], []
    for _ in range(3):
        dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        M.xw_replicate(X, Wt, rep, sync=False)
        e1.record(stream)
        torch.cuda.synchronize(dev)
        dist.barrier()
        fused.append(e0.elapsed_time(e1))
        dist.barrier()
        e0.record(stream)
        M.xw_bf16(X, Wt, out=full[rank * per: rank * per + (r1 - r0)])
        if nccl:
            dist.all_gather_into_tensor(full, full[rank * per:(rank + 1) * per])
        else:           # gloo (several ranks sharing one GPU in tests): host staging
            host = torch.empty(full.shape, dtype=full.dtype)
            dist.all_gather_into_tensor(host, full[rank * per:(rank + 1) * per].cpu())
            full.copy_(host)
        e1.record(stream)
        torch.cuda.synchronize(dev)
        unfused.append(e0.elapsed_time(e1))
    ok = torch.equal(rep.B, full[: g.n])
    t = torch.tensor([min(fused), min(unfused), 0.0 if ok else 1.0], dtype=torch.float64,
                     device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    rep.close()
    return {"F": F, "fused_xw_bcast_ms": float(t[0]),
            ("xw_then_nccl_allgather_ms" if nccl else "xw_then_gloo_allgather_ms"): float(t[1]),
            "replicas_equal": bool(t[2] == 0.0)}


def gcn_layer_pipelined(M, g, K, rank, world, dev):
    """NEXT-3 multi-GPU: one aggregation layer A*(X*W) from row-sharded X.  pipelined:
    ShardedGCNLayer (combination + replication per column tile overlapped with the
    sharded SpMM of the tiles already resident); serial: the whole replication, a
    barrier, then the SpMM.  CUDA events, max over ranks, best of 3."""
    import torch
    import torch.distributed as dist
    F = FEATURES.get(g.name.split("-")[0], 64)
    ldx = -(-F // 8) * 8
    layer = M.ShardedGCNLayer(g.row_ptr, g.col_idx, g.val, g.n, F, K, rank, world, dev,
                              tile_cols=64)
    gen = torch.Generator(device="cpu").manual_seed(1000 + rank)
    X = torch.zeros((max(layer.r1 - layer.r0, 1), ldx), dtype=torch.bfloat16)
    X[:, :F] = torch.randn(X.shape[0], F, generator=gen).to(torch.bfloat16)
    X = X.to(dev)[: layer.r1 - layer.r0, :F]
    Wt = torch.zeros((K, ldx), dtype=torch.bfloat16)
    Wt[:, :F] = torch.randn(K, F, generator=torch.Generator().manual_seed(7)) / F ** 0.5
    Wt = Wt.to(dev)[:, :F]
    s_xw, s_agg = torch.cuda.Stream(dev), torch.cuda.current_stream(dev)
    pipe, serial = [], []
    for _ in range(4):
        dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s_agg)
        layer(X, Wt, s_xw=s_xw, s_agg=s_agg)
        e1.record(s_agg)
        torch.cuda.synchronize(dev)
        pipe.append(e0.elapsed_time(e1))
        dist.barrier()
        e0.record(s_agg)
        layer.replicate(X, Wt, s_agg)             # same kernels on one stream: every tile
        for slot in range(len(layer.tiles)):      # replicated before any SpMM
            layer.aggregate_tile(slot, s_agg)
        e1.record(s_agg)
        torch.cuda.synchronize(dev)
        serial.append(e0.elapsed_time(e1))
    t = torch.tensor([min(pipe[1:]), min(serial[1:])], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    layer.close()
    return {"F": F, "tile_cols": layer.tile, "pipelined_ms": float(t[0]),
            "serial_ms": float(t[1])}


def agreed(fn, dev):
    """Run fn() on every rank, then agree on the outcome with one all_reduce: the result
    when every rank succeeded, else {"error": ...} on every rank."""
    import torch
    import torch.distributed as dist
    res, err = None, None
    try:
        res = fn()
    except Exception as e:  # pragma: no cover
        err = str(e)[:200]
    ok = torch.tensor([0 if err else 1], device=dev)
    dist.all_reduce(ok, op=dist.ReduceOp.MIN)
    if int(ok[0]) == 1:
        return res
    return {"error": err or "failed on another rank"}


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
        return
    world_env = int(os.environ.get("WORLD_SIZE", "1"))
    if world_env > 1 and "OMP_NUM_THREADS" not in os.environ:
        # every rank generates the same graph on the host: share the cores
        local_world = int(os.environ.get("LOCAL_WORLD_SIZE", world_env))
        os.environ["OMP_NUM_THREADS"] = str(max(1, (os.cpu_count() or 1) // local_world))
    import torch
    import torch.distributed as dist
    import graphgen as G
    import paper_conf_ispass_shangndk23_b200 as M
    from paper_conf_ispass_shangndk23_b200 import _lib as L
    from paper_conf_ispass_shangndk23_b200.api import _p, _stream, FIXUP

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    ngpu = torch.cuda.device_count()
    dev = torch.device("cuda", local % ngpu)   # several ranks may share a GPU (gloo tests)
    torch.cuda.set_device(dev)
    if world > 1:
        import datetime
        # a rank that dies makes torchrun tear the job down; a collective that waits for
        # a rank stuck elsewhere errors out after this long instead of hanging
        tmo = datetime.timedelta(seconds=600)
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=dev, timeout=tmo)
        else:
            dist.init_process_group("gloo", timeout=tmo)

    name = args.workload
    K = args.K or G.WORKLOADS[name][3][0]
    tdtype = torch.bfloat16 if args.dtype == "bf16" else torch.float32
    b_elt = 2 if args.dtype == "bf16" else 4
    dt_code = L.MPS_DT_BF16 if args.dtype == "bf16" else L.MPS_DT_F32
    fix = FIXUP[args.fixup]

    t0 = time.perf_counter()
    g = G.workload(name)
    Bh = G.features(name, K)
    gen_s = time.perf_counter() - t0

    stream = torch.cuda.current_stream(dev)
    s_ptr = _stream(stream)
    Bd = torch.from_numpy(Bh).to(dev).to(tdtype)
    l2 = torch.cuda.get_device_properties(dev).L2_cache_size
    flush = torch.empty(2 * l2 // 4 + 1024, dtype=torch.float32, device=dev)
    flush_sink = torch.empty(1, dtype=torch.float32, device=dev)

    flush_clean = torch.zeros_like(flush) if args.flush == "write" else None

    def do_flush():
        if args.flush == "write":
            # write 2x L2, then read another 2x L2: the written lines are evicted (and
            # written back) here, untimed, so the step starts from a cold L2 holding
            # clean lines instead of paying the flush's write-backs
            flush.zero_()
            torch.sum(flush_clean, dim=0, out=flush_sink[0])
        elif args.flush == "read":
            torch.sum(flush, dim=0, out=flush_sink[0])

    launches_per_step = 0
    seg_ms = []
    step_ms = []
    part_ms = []

    if world == 1:
        A = M.CSR.from_numpy(g.row_ptr, g.col_idx, g.val, g.n, device=dev)
        a = A.struct()
        # the path of record: mps_partition_split (a2 + cut-row zeroing) then
        # mps_spmm_segments_hot (a3 + a4), events between them (api.OnlineStep; the
        # full-size parity tests run exactly this object)
        online = M.OnlineStep(A, K, b_dtype=tdtype, fixup=args.fixup,
                              items_per_part=args.items_per_part, min_parts=args.min_parts,
                              hot=args.hot)
        P, Lp = online.P, online.L
        C = online.C
        hot_rows = online.hot_rows
        launches_per_step = online.launches(l2)

        def step(ev=None):
            online(Bd, events=ev)
        units_nnz = g.nnz
        units_rows = g.m
    else:
        # B replication over NVLink (offline, reported separately, not in the step)
        per = -(-g.n // world)
        Bmine = Bd[rank * per: min(g.n, (rank + 1) * per)].contiguous()
        rep_ms = []
        for _ in range(3):
            dist.barrier()
            r0, r1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            r0.record(stream)
            Brep = M.replicate_B(Bmine, g.n, world)
            r1.record(stream)
            torch.cuda.synchronize(dev)
            rep_ms.append(r0.elapsed_time(r1))
        assert torch.equal(Brep, Bd)
        b_rep = torch.tensor([min(rep_ms)], dtype=torch.float64, device=dev)
        dist.all_reduce(b_rep, op=dist.ReduceOp.MAX)
        b_rep_ms = float(b_rep[0])
        del Brep
        # NEXT-3 extras (--extras; off by default so that the scaling run's line cannot
        # be lost to them): the combination fused with the replication, and one
        # pipelined GCN layer.  Each is entered by every rank and ends in one all_reduce
        # of its status, so all ranks agree on the outcome before any later collective.
        xw_rep = gcn_layer = None
        if args.extras and K % 16 == 0 and 16 <= K <= 256:
            xw_rep = agreed(lambda: xw_replication(M, g, K, rank, world, dev, stream), dev)
            if world <= 16:
                gcn_layer = agreed(lambda: gcn_layer_pipelined(M, g, K, rank, world, dev), dev)
        sh_kw = dict(b_dtype=tdtype, fixup=args.fixup, items_per_part=args.items_per_part,
                     min_parts=args.min_parts)
        # the rank's shard (local work only: no collective inside)
        sh = M.ShardedSpMM(g.row_ptr, g.col_idx, g.val, g.n, K, rank, world, dev, **sh_kw)
        tails_mode = "nccl"
        if args.tails in ("auto", "p2p") and world <= 16:
            # mailboxes over CUDA IPC: enable_p2p maps every peer and agrees across ranks
            # (one all_reduce) before returning, so it succeeds or raises on ALL ranks
            try:
                sh.enable_p2p()
                tails_mode = "p2p"
            except Exception as e:  # uniform across ranks
                print("p2p tails unavailable (rank %d): %s" % (rank, e), file=sys.stderr)
        if tails_mode == "p2p":
            # cross-check one step of each exchange before trusting the fused one
            sh.local(Bd)
            sh.settle(M.exchange_tails(sh.tail, world))
            ref_rows = sh.C[: sh.rows].clone()
            sh.local_p2p(Bd)
            torch.cuda.synchronize(dev)
            # the two runs differ only in fp32 atomic order: compare against the scale of C
            scale = float(ref_rows.abs().max()) if ref_rows.numel() else 0.0
            same = torch.allclose(sh.C[: sh.rows], ref_rows, rtol=1e-4, atol=1e-5 * scale + 1e-30)
            ok = torch.tensor([1 if same else 0], device=dev)
            dist.all_reduce(ok, op=dist.ReduceOp.MIN)
            del ref_rows
            if int(ok[0]) != 1:
                tails_mode = "nccl"
        P, Lp = None, None
        tiles = n_tiles(g.n, K, b_elt, l2)
        launches_per_step = 1 + tiles * (2 if fix == L.MPS_FIXUP_CARRY else 1) + \
            (0 if tails_mode == "p2p" else 1)

        def step(ev=None):
            if ev is not None:
                ev[0].record(stream)
            if tails_mode == "p2p":       # exchange fused into the final kernel (peer memory)
                sh.local_p2p(Bd)
                if ev is not None:
                    ev[1].record(stream)
                return
            sh.local(Bd)
            if ev is not None:
                ev[1].record(stream)
            tails = M.exchange_tails(sh.tail, world)      # the path's one collective
            sh.settle(tails)
        units_nnz = g.nnz
        units_rows = g.m

    def barrier():
        if world > 1:
            dist.barrier()

    # warm-up (untimed)
    for _ in range(max(args.warmup, 0)):
        do_flush()
        step()
    torch.cuda.synchronize(dev)

    run_step = step
    if args.cuda_graph and world == 1:
        C_eager = C.clone() if world == 1 else None
        cg = torch.cuda.CUDAGraph()
        with torch.cuda.graph(cg):
            step()
        torch.cuda.synchronize(dev)
        C.fill_(float("nan"))
        cg.replay()
        torch.cuda.synchronize(dev)
        # a replay must reproduce the eager step (an empty capture would leave the NaNs)
        scale = float(C_eager.abs().max()) if C_eager.numel() else 0.0
        if not torch.allclose(C, C_eager, rtol=1e-4, atol=1e-5 * scale + 1e-30):
            raise RuntimeError("CUDA-graph replay does not reproduce the eager step")
        del C_eager

        def run_step(ev=None):            # events cannot split a replay: time the graph
            cg.replay()
        stream = torch.cuda.current_stream(dev)

    small_path = world == 1 and online.path == L.MPS_PATH_SMALL_FUSED
    if world == 1:
        launches_per_step = online.launches(l2)    # the path is resolved by the warm-up
    path_desc = ("small_fused (1 kernel + carry reduction)" if small_path else
                 "partition+segments") if world == 1 else "sharded"
    inner_events = not (args.cuda_graph and world == 1) and not small_path
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True),
            torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
           for _ in range(args.steps)]
    clocks = ClockSampler(dev.index)
    clocks.start()
    time.sleep(0.3)
    barrier()
    torch.cuda.synchronize(dev)
    wall0 = time.perf_counter()
    for i in range(args.steps):
        do_flush()                        # L2 flush between timed steps (not timed)
        evs[i][0].record(stream)
        # inner events (around the segment kernel, for its live roofline) only where the
        # step has a separate segment kernel to time; each event record costs ~2.5 us of
        # stream time, which would otherwise inflate the tiny graphs' steps
        run_step((evs[i][1], evs[i][2]) if inner_events else None)
        evs[i][3].record(stream)
        # each step runs alone on the GPU (the protocol of the cuSPARSE reference point:
        # flush, event, call, event, synchronise); for the tiny graphs the launch of a
        # step queued behind the previous one otherwise adds several microseconds
        torch.cuda.synchronize(dev)
    torch.cuda.synchronize(dev)
    barrier()
    wall = time.perf_counter() - wall0
    clk = clocks.stop()
    for e in evs:
        step_ms.append(e[0].elapsed_time(e[3]))
        if inner_events:
            seg_ms.append(e[1].elapsed_time(e[2]))
            part_ms.append(e[0].elapsed_time(e[1]))
        else:                             # the whole step is the timed kernel sequence
            seg_ms.append(e[0].elapsed_time(e[3]))
            part_ms.append(0.0)
    t_step = float(np.mean(step_ms))
    t_seg = float(np.mean(seg_ms))
    # parity of the C the timed steps produced (untimed): sampled rows -- every row cut
    # by a merge-path boundary, random rows, the longest rows -- against the fp64 oracle
    # within the north-star tolerance, and all column sums; a mismatch fails the run
    if world == 1:
        parity = validate_output(g, Bd, C, online.cx, online.cy, K)
    else:
        parity = validate_output_shard(g, Bd, sh, K, rank)
        pt = torch.tensor([1.0 if parity["ok"] else 0.0], dtype=torch.float64, device=dev)
        dist.all_reduce(pt, op=dist.ReduceOp.MIN)
        parity["all_ranks_ok"] = bool(pt[0] == 1.0)
    if world > 1:
        tt = torch.tensor([t_step, t_seg], dtype=torch.float64, device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        t_step, t_seg = float(tt[0]), float(tt[1])

    flops = 2.0 * units_nnz * K
    gflops = flops / (t_step * 1e-3) / 1e9
    bytes_alg = alg_bytes(units_rows, units_nnz, K, b_elt)
    hbm_peak, peak_src = peaks()
    eff_gbs = bytes_alg / (t_step * 1e-3) / 1e9

    # dominant kernel roofline: the a3 segment kernel (per-rank algorithmic bytes)
    if world == 1:
        seg_bytes = bytes_alg
    else:
        y0, y1 = int(sh.Y[rank]), int(sh.Y[rank + 1])
        seg_bytes = alg_bytes(sh.rows, y1 - y0, K, b_elt)
    seg_gbs = seg_bytes / (t_seg * 1e-3) / 1e9
    traffic = None          # ncu DRAM bytes per launch of the segment kernel
    units = None
    prof = os.path.join(ROOT, "profiles", "traffic.json")
    key = "%s-k%d-%s-%s" % (name, K, args.dtype, "atomic" if args.fixup == "auto" else args.fixup)
    if os.path.exists(prof) and world == 1:
        with open(prof) as f:
            tj = json.load(f)
            traffic_step = tj.get(key)          # DRAM bytes of all column tiles of a step
            if isinstance(traffic_step, (int, float)):
                # per launch, like `achieved` (one launch = one column tile)
                traffic = int(traffic_step / max(1, n_tiles(g.n, K, b_elt, l2)))
            u = tj.get("_units", {}).get(key)
            if u:   # ncu of the same kernel: which unit binds (B in L2 -> L2, else DRAM)
                units = dict(u, source="ncu --set full (profiles/traffic.json: %s)"
                             % tj.get("_note", "")[:60],
                             note=("B fits in L2: the algorithmic-byte fraction exceeds 1; "
                                   "the binding unit is L2 (lts_throughput_pct)")
                             if b_elt * g.n * K <= 0.5 * l2 else
                             "B exceeds L2: DRAM-bound gathers (dram traffic above)")

    # live L2 probes (tools/l2_probe.cu): where B fits in L2 the gathers are bound by
    # L2 -> SM bandwidth.  "lean_gather_256B" (power-of-two table, one IMAD per row
    # index, 16 gathers of 16 B in flight per lane) is the L2 read ceiling the roofline
    # uses; the older hashed gather and the streaming reads are reported beside it.
    l2_peak, l2_src = None, None
    if world == 1 and not args.no_l2_probe:
        try:
            import __graft_entry__
            lp = ctypes.CDLL(__graft_entry__.build_l2_probe())
            res = {}
            for mode, key in ((2, "lean_gather_256B"), (3, "lean_stream"), (0, "gather_256B"),
                              (1, "stream")):
                gb, pm = ctypes.c_float(), ctypes.c_float()
                rc = lp.l2_probe_read_gbs2(ctypes.c_int64(48 << 20), ctypes.c_int32(256),
                                           ctypes.c_int32(mode), ctypes.byref(gb),
                                           ctypes.byref(pm))
                if rc == 0:
                    res[key] = round(gb.value, 1)
            torch.cuda.synchronize(dev)
            if res:
                units = dict(units or {})
                units["l2_probe_gbs"] = res
                units["l2_probe_source"] = ("measured live: tools/l2_probe.cu, 48 MB "
                                            "L2-resident table, 16-B no-L1 loads, best of 4 "
                                            "grid shapes")
                l2_peak = max(res.values())
                l2_src = "live L2 probe (max of %s)" % ", ".join(sorted(res))
                units["segment_vs_l2_probe"] = seg_gbs / l2_peak
        except Exception as e:  # pragma: no cover
            units = dict(units or {}, l2_probe_error=str(e)[:200])
    # binding unit of the segment kernel: L2 when a column tile's gathered B slice fits
    # in half the L2 (its rows stay resident), HBM otherwise
    tile_cols = min(K, n_tile_cols(g.n, K, b_elt, l2))
    b_slice = b_elt * g.n * tile_cols
    if b_slice <= 0.5 * l2:
        if l2_peak is None:
            l2_peak, l2_src = L2_PEAK_FALLBACK_GBS, L2_PEAK_FALLBACK_SRC
        roof = {"bound": "l2", "achieved": seg_gbs, "peak": l2_peak, "unit": "GB/s",
                "frac": seg_gbs / l2_peak, "peak_source": l2_src,
                "why": "B column slice (%.1f MB) <= L2/2: gathers hit L2; every byte of the "
                       "algorithmic count crosses L2 -> SM" % (b_slice / 1e6)}
    else:
        roof = {"bound": "hbm", "achieved": seg_gbs, "peak": hbm_peak, "unit": "GB/s",
                "frac": seg_gbs / hbm_peak, "peak_source": peak_src,
                "why": "B column slice (%.1f MB) > L2/2: gathers miss L2" % (b_slice / 1e6)}
        if isinstance(traffic, (int, float)) and traffic > 0:
            # ncu DRAM bytes of one launch (one column tile) over the live launch time
            per_launch_s = t_seg * 1e-3 / max(1, n_tiles(g.n, K, b_elt, l2))
            roof["dram_frac_of_peak_ncu_bytes"] = traffic / per_launch_s / 1e9 / hbm_peak
    # The workload's own gather stream replayed alone (tools/gather_replay.cu): the B-row
    # gathers of every non-zero in CSR order (row col_idx[j] of each column tile), read
    # with nothing else in the way, L2 flushed first.  Its time is the attainable time of
    # the kernel's dominant traffic on this box, with the L2-hit / DRAM-miss mix the real
    # column pattern produces; roofline.peak is the algorithmic byte rate at that time.
    row_bytes = tile_cols * b_elt
    if world == 1 and not args.no_l2_probe and row_bytes in (64, 128, 256, 512) \
            and not small_path:
        try:
            import __graft_entry__
            gr = ctypes.CDLL(__graft_entry__.build_gather_replay())
            gms, gby = ctypes.c_float(), ctypes.c_double()
            rc = gr.gather_replay(_p(A.col_idx), ctypes.c_int64(g.nnz), _p(Bd),
                                  ctypes.c_int32(row_bytes), ctypes.c_int64(K * b_elt),
                                  ctypes.c_int32(3), ctypes.byref(gms), ctypes.byref(gby))
            torch.cuda.synchronize(dev)
            if rc == 0 and gms.value > 0:
                tiles = n_tiles(g.n, K, b_elt, l2)
                t_rep = gms.value * tiles                       # every column tile
                roof["attainable"] = {
                    "what": "gather replay: the B-row gathers of the workload's own col_idx "
                            "stream alone, %d x %d-B rows per non-zero, L2 flushed" % (
                                tiles, row_bytes),
                    "replay_ms": t_rep, "segment_ms": t_seg,
                    "gather_gbs": gby.value * tiles / (t_rep * 1e-3) / 1e9,
                    "frac": t_rep / t_seg}
                roof["units_frac_against"] = {"l2_probe": (seg_gbs / l2_peak) if l2_peak else None,
                                              "hbm_peak": seg_gbs / hbm_peak}
                roof.update({"peak": seg_bytes / (t_rep * 1e-3) / 1e9, "frac": t_rep / t_seg,
                             "peak_source": "gather replay of this workload (roofline.attainable)"})
                # the same replay at the fp32 kernel's own register-resident depth (3 CTAs
                # x 8 warps, 8 x 16-B gathers per lane; the deep-gather kernel: 2 CTAs, 16):
                # what the gather stream alone takes with the bytes in flight the kernel
                # can hold -- a diagnostic beside the attainable replay, not the peak
                if b_elt == 4 and row_bytes == 256:
                    deep = g.nnz >= 32 * g.n and g.n * row_bytes > 0.5 * l2
                    psm, ul = (2, 0) if deep else (3, 8)
                    sms, sby = ctypes.c_float(), ctypes.c_double()
                    rc2 = gr.gather_replay_cfg(_p(A.col_idx), ctypes.c_int64(g.nnz), _p(Bd),
                                               ctypes.c_int32(row_bytes), ctypes.c_int64(K * b_elt),
                                               ctypes.c_int32(3), ctypes.c_int32(psm),
                                               ctypes.c_int32(ul), ctypes.byref(sms),
                                               ctypes.byref(sby))
                    torch.cuda.synchronize(dev)
                    if rc2 == 0 and sms.value > 0:
                        roof["attainable"]["same_depth"] = {
                            "what": "the same replay with the kernel's bytes in flight: %d CTAs "
                                    "x 8 warps per SM, %d x 16-B gathers per lane" % (
                                        psm, ul or 16),
                            "replay_ms": sms.value * tiles, "frac": sms.value * tiles / t_seg}
        except Exception as e:  # pragma: no cover
            roof["attainable_error"] = str(e)[:200]

    # cuSPARSE on the same A, B (reference point; not the product)
    cus = None
    if world == 1 and args.dtype == "f32" and not args.no_cusparse:
        try:
            import __graft_entry__
            cl = ctypes.CDLL(__graft_entry__.build_cusparse_ref())
            bm, ba = ctypes.c_float(), ctypes.c_int()
            per = (ctypes.c_float * 4)()
            Cc = torch.empty((g.m, K), dtype=torch.float32, device=dev)
            rc = cl.cusparse_spmm_best(ctypes.c_int64(g.m), ctypes.c_int64(g.n),
                                       ctypes.c_int64(g.nnz), _p(A.row_ptr), _p(A.col_idx),
                                       _p(A.val), _p(Bd), ctypes.c_int64(K), ctypes.c_int32(K),
                                       _p(Cc), ctypes.c_int64(K), ctypes.c_int(5),
                                       ctypes.byref(bm), ctypes.byref(ba), per)
            torch.cuda.synchronize(dev)
            if rc == 0:
                names = ["ALG_DEFAULT", "CSR_ALG1", "CSR_ALG2", "CSR_ALG3"]
                cus = {"ms": bm.value, "gflops": 2.0 * g.nnz * K / (bm.value * 1e-3) / 1e9,
                       "best_alg": names[ba.value],
                       "ms_per_alg": {names[i]: (round(per[i], 4) if per[i] >= 0 else None)
                                      for i in range(4)},
                       "l2": "flushed before every call", "note": "library SpMM, context only"}
            else:
                cus = {"error": "cusparse rc %d" % rc}
            del Cc
        except Exception as e:  # pragma: no cover
            cus = {"error": str(e)[:200]}

    # end to end with the graph resident (offline setting): B host -> device,
    # online SpMM, C device -> host, through mps_spmm_host_dense (context for e2e below)
    e2e_res = None
    if world == 1 and args.e2e_steps > 0:
        Bh_r = torch.from_numpy(Bh).to(tdtype).pin_memory()
        Ch_r = torch.empty((g.m, K), dtype=torch.float32).pin_memory()
        nbr = ctypes.c_size_t()
        L.mps_spmm_host_dense_workspace_bytes(ctypes.byref(a), K, dt_code, K, K,
                                              args.items_per_part, args.min_parts, fix,
                                              ctypes.byref(nbr))
        wsr = torch.empty(nbr.value, dtype=torch.uint8, device=dev)

        def res_step():
            L.mps_spmm_host_dense(ctypes.byref(a), _p(Bh_r), dt_code, K, K, _p(Ch_r), K,
                                  args.items_per_part, args.min_parts, fix, _p(wsr), nbr.value,
                                  s_ptr)
        res_step()
        torch.cuda.synchronize(dev)
        r_ms = []
        for _ in range(args.e2e_steps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            res_step()
            e1.record(stream)
            torch.cuda.synchronize(dev)
            r_ms.append(e0.elapsed_time(e1))
        t_res = float(np.mean(r_ms))
        e2e_res = {"value": flops / (t_res * 1e-3) / 1e9, "unit": "GFLOP/s",
                   "h2d_bytes_per_step": int(b_elt * g.n * K),
                   "d2h_bytes_per_step": int(4 * g.m * K), "ms_per_step": t_res,
                   "path": "mps_spmm_host_dense (A resident on the device; pinned host B -> C)"}
        del wsr, Bh_r, Ch_r

    # end-to-end through the public C ABI on pinned HOST buffers (rank 0 layout, N=1)
    e2e = None
    if world == 1 and args.e2e_steps > 0:
        pin = lambda x: torch.from_numpy(x).pin_memory()
        rp_h, ci_h, va_h = pin(g.row_ptr), pin(g.col_idx), pin(g.val)
        Bh_t = torch.from_numpy(Bh).to(tdtype).pin_memory()
        Ch = torch.empty((g.m, K), dtype=torch.float32).pin_memory()
        from paper_conf_ispass_shangndk23_b200.api import host_workspace_bytes
        nbh = host_workspace_bytes(rp_h, ci_h, va_h, g.n, Bh_t, Ch, args.items_per_part,
                                   args.min_parts, args.fixup)
        wsh = torch.empty(nbh, dtype=torch.uint8, device=dev)
        del A, C, online, flush
        torch.cuda.empty_cache()
        ah = M.mps_csr_host(rp_h, ci_h, va_h, g.n)

        def e2e_step():
            L.mps_spmm_host(ctypes.byref(ah), _p(Bh_t), dt_code, K, K, _p(Ch), K,
                            args.items_per_part, args.min_parts, fix, _p(wsh), nbh, s_ptr)
        e2e_step()
        torch.cuda.synchronize(dev)
        e_ms = []
        for _ in range(args.e2e_steps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            e2e_step()
            e1.record(stream)
            torch.cuda.synchronize(dev)
            e_ms.append(e0.elapsed_time(e1))
        t_e2e = float(np.mean(e_ms))
        h2d = 4 * (g.m + 1) + 8 * g.nnz + b_elt * g.n * K
        d2h = 4 * g.m * K
        e2e = {"value": flops / (t_e2e * 1e-3) / 1e9, "unit": "GFLOP/s",
               "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
               "ms_per_step": t_e2e, "path": "mps_spmm_host (pinned host A, B -> C)"}
        # the e2e ceiling: pinned H2D bandwidth of this box, measured on the step's own
        # pinned col_idx buffer (one warm-up, best of 3)
        try:
            dp = torch.empty(ci_h.numel(), dtype=ci_h.dtype, device=dev)
            best = 1e9
            for i in range(4):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                dp.copy_(ci_h, non_blocking=True)
                e1.record(stream)
                torch.cuda.synchronize(dev)
                if i:
                    best = min(best, e0.elapsed_time(e1))
            h2d_gbs = ci_h.numel() * ci_h.element_size() / (best * 1e-3) / 1e9
            e2e["h2d_gbs_measured"] = round(h2d_gbs, 2)
            e2e["h2d_bound_ms"] = h2d / h2d_gbs / 1e6
            e2e["frac_of_h2d_bound"] = e2e["h2d_bound_ms"] / t_e2e
            del dp
        except Exception as e:  # pragma: no cover
            e2e["h2d_probe_error"] = str(e)[:200]

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        try:
            rate, cores, sample, _ = cpu_oracle_rate(g, Bh if args.dtype == "f32" else
                                                     Bd.float().cpu().numpy(), K,
                                                     args.cpu_seconds)
            cpu = {"value": rate, "unit": "GFLOP/s", "cores": cores, "kind": "oracle",
                   "sample": sample}
        except Exception as e:  # pragma: no cover
            cpu = {"value": None, "unit": "GFLOP/s", "cores": None, "kind": "oracle",
                   "sample": "failed: %s" % e}

    if rank == 0:
        line = {
            "metric": METRIC,
            "value": gflops,
            "unit": "GFLOP/s",
            "n_gpus": world,
            "steps": args.steps,
            "warmup": args.warmup,
            "ms_per_step": t_step,
            "higher_is_better": True,
            "scaling": "strong",
            "vs_baseline": None,
            "dtype": "f32" if args.dtype == "f32" else "bf16-in/f32-acc",
            "data": "synthetic",
            "config": {
                "workload": "%s-k%d" % (name, K), "graph": g.name, "n": g.m, "nnz": g.nnz,
                "K": K, "b_dtype": args.dtype, "fixup": args.fixup,
                "path": path_desc,
                "num_parts": P, "items_per_part": Lp, "mode": "online (partition every step)",
                "timing": "CUDA events around each step on the launching stream, every step "
                          "synchronised (the cuSPARSE reference's protocol); value = mean",
                "l2": {"write": "flushed before every timed step (2x L2 write, then 2x L2 read "
                                 "of a second buffer so no dirty lines remain; untimed)",
                       "read": "flushed before every timed step (2x L2 read, untimed)",
                       "none": "not flushed (col/val > L2)"}[args.flush],
                "parallelism": "merge-path shards x%d" % world, "graph_sha": g.digest(),
                "tail_exchange": (tails_mode if world > 1 else None),
                "cuda_graph": bool(args.cuda_graph and world == 1),
                "hot_rows": (hot_rows if world == 1 else None),
                "gen_s": round(gen_s, 2),
            },
            "effective_gbs": eff_gbs,
            "hbm_frac_step": eff_gbs / hbm_peak,
            "partition_zero_ms": float(np.mean(part_ms)),
            "segment_ms": t_seg,
            "segment_ms_steps": [round(x, 4) for x in seg_ms],
            "step_ms_p10_p90": [float(np.percentile(step_ms, 10)),
                                float(np.percentile(step_ms, 90))],
            "step_ms_min_median": [float(np.min(step_ms)), float(np.median(step_ms))],
            "wall_s_timed_region": wall,
            "roofline": dict(roof, kernel="segment_kernel (a3)", traffic=traffic,
                             algorithmic_bytes_per_launch=int(seg_bytes), units=units),
            # the north-star figure: algorithmic bytes of the step against HBM, which
            # exceeds 1 where B is L2-resident
            "north_star_hbm": {"achieved": eff_gbs, "peak": hbm_peak, "unit": "GB/s",
                               "frac": eff_gbs / hbm_peak, "bar": 0.6 * 8000.0 / hbm_peak,
                               "peak_source": peak_src},
            "parity": parity,
            "b_replication": ({"ms": b_rep_ms, "bytes_per_rank_received": int(
                (world - 1) * (-(-g.n // world)) * K * b_elt), "collective": "all_gather_into_tensor",
                "in_step": False, "fused_xw": xw_rep,
                "gcn_layer_bf16": gcn_layer} if world > 1 else None),
            "cpu_baseline": cpu,
            "e2e": e2e,
            "e2e_graph_resident": e2e_res,
            "cusparse": cus,
            "paper_context": PAPER_CONTEXT,
            "gpu_launches": int(launches_per_step * args.steps),
            "clocks": clk,
        }
        s = json.dumps(line)
        print(s, flush=True)
        if args.out:
            with open(args.out, "a") as f:
                f.write(s + "\n")
    if world > 1:
        dist.destroy_process_group()
    if not parity["ok"] or not parity.get("all_ranks_ok", True):
        print("bench.py: the timed step's C fails the oracle check: %s" % json.dumps(parity),
              file=sys.stderr)
        sys.exit(3)


if __name__ == "__main__":
    main()
