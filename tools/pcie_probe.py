"""Pinned host -> device and device -> host copy bandwidth (one 1 GB cudaMemcpyAsync and
64 x 16 MB chunks), the ceiling of the e2e line.  python tools/pcie_probe.py"""
import torch, time
n = 1 << 30
h = torch.empty(n, dtype=torch.uint8).pin_memory()
d = torch.empty(n, dtype=torch.uint8, device="cuda")
s = torch.cuda.current_stream()
def t(fn, reps=5):
    fn(); torch.cuda.synchronize()
    best = 1e9
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return n / (best * 1e-3) / 1e9
print("H2D 1 GB     GB/s %.1f" % t(lambda: d.copy_(h, non_blocking=True)))
print("D2H 1 GB     GB/s %.1f" % t(lambda: h.copy_(d, non_blocking=True)))
c = 16 << 20
def chunks():
    for i in range(0, n, c):
        d[i:i + c].copy_(h[i:i + c], non_blocking=True)
print("H2D 16 MB x64 GB/s %.1f" % t(chunks))
