"""Launch-latency floor of the tiny-graph step timing protocol (bench.py --cuda-graph):
L2 flushed (2x L2 write + 2x L2 read of another buffer) before each step, CUDA events
around the step on the stream.  Steps: a graph of 1 or 2 trivial library kernels, the
small-graph fused online step (graph and eager), the two-kernel online step, and each
kernel of the fused step alone (MPS_SMALL_SKIP_REDUCE-free: timed by events between)."""
import ctypes, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np, torch
import graphgen as G
import paper_conf_ispass_shangndk23_b200 as M
from paper_conf_ispass_shangndk23_b200 import _lib as L
from paper_conf_ispass_shangndk23_b200.api import _p, _stream

dev = torch.device("cuda", 0)
l2 = torch.cuda.get_device_properties(dev).L2_cache_size
fl = torch.empty(2 * l2 // 4 + 1024, device=dev)
fc = torch.zeros_like(fl)
sink = torch.empty(1, device=dev)


def flush():
    fl.zero_()
    torch.sum(fc, dim=0, out=sink[0])


def timeit(fn, n=40, graph=True):
    fn(); torch.cuda.synchronize()
    run = fn
    if graph:
        cg = torch.cuda.CUDAGraph()
        with torch.cuda.graph(cg):
            fn()
        run = cg.replay
    ts = []
    st = torch.cuda.current_stream()
    for _ in range(n):
        flush()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st); run(); e1.record(st)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    ts = np.array(ts[3:])
    return {"mean_us": round(float(ts.mean()), 2), "median_us": round(float(np.median(ts)), 2),
            "min_us": round(float(ts.min()), 2)}


x = torch.zeros((1, 8), device=dev)
h = torch.zeros((1, 8), dtype=torch.bfloat16, device=dev)
def one():
    L.mps_relu_to_bf16(_p(x), 1, 8, 8, _p(h), 8, _stream())
def two():
    one(); one()
res = {"graph_1_trivial_kernel": timeit(one), "graph_2_trivial_kernels": timeit(two),
       "eager_1_trivial_kernel": timeit(one, graph=False),
       "eager_2_trivial_kernels": timeit(two, graph=False)}
for wl, K in (("cora", 16), ("pubmed", 16), ("pubmed", 64)):
    g = G.workload(wl)
    A = M.CSR.from_numpy(g.row_ptr, g.col_idx, g.val, g.n)
    B = torch.from_numpy(G.features(wl, K)).to(dev)
    for fx in ("auto", "atomic"):
        st = M.OnlineStep(A, K, fixup=fx)
        key = "%s-k%d-%s" % (wl, K, "small_fused" if fx == "auto" else "partition+segments")
        res[key + "-graph"] = timeit(lambda: st(B))
        res[key + "-eager"] = timeit(lambda: st(B), graph=False)
    cl = ctypes.CDLL(os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "libcusparse_ref.so"))
    bm, ba = ctypes.c_float(), ctypes.c_int()
    per = (ctypes.c_float * 4)()
    Cc = torch.empty((g.m, K), device=dev)
    cl.cusparse_spmm_best(ctypes.c_int64(g.m), ctypes.c_int64(g.n), ctypes.c_int64(g.nnz),
                          _p(A.row_ptr), _p(A.col_idx), _p(A.val), _p(B), ctypes.c_int64(K),
                          ctypes.c_int32(K), _p(Cc), ctypes.c_int64(K), ctypes.c_int(20),
                          ctypes.byref(bm), ctypes.byref(ba), per)
    res["%s-k%d-cusparse_eager_best_of_20" % (wl, K)] = round(bm.value * 1e3, 2)
for k, v in res.items():
    print(k, json.dumps(v))
