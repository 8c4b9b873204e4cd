"""NEXT-3 multi-GPU: B = X*W fused with the replication of B (mps_xw_bf16_bcast).

1. Loopback on one GPU: G "ranks" each write their row block into G local replicas;
   every replica must equal B = X*W (integer inputs: exact; the fp64 product is the
   reference, no CUDA value is used as an expected value).
2. Two processes on one GPU (gloo process group, CUDA IPC between the processes): the
   real PeerReplicas / xw_replicate path, each process mapping the other's replica.
"""
import os
import re
import socket
import subprocess
import sys

import numpy as np
import pytest
import torch

import oracle as O

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

if torch.cuda.is_available():
    import paper_conf_ispass_shangndk23_b200 as M
    from paper_conf_ispass_shangndk23_b200.api import _p, _stream


def _int_inputs(n, F, N, seed):
    g = torch.Generator(device="cpu").manual_seed(seed)
    X = torch.randint(-1, 2, (n, F), generator=g).to(torch.bfloat16)
    W = torch.randint(-1, 2, (F, N), generator=g).to(torch.bfloat16)
    return X, W, torch.from_numpy(O.xw_f64(X.float().numpy(), W.float().numpy()))  # exact


@pytest.mark.parametrize("G", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("N", [16, 64, 128, 256])
def test_xw_bcast_loopback(G, N):
    import ctypes
    n, F = 1000 + 3 * N + 77, 72
    X, W, ref = _int_inputs(n, F, N, seed=G * 100 + N)
    Xd, Wt = X.cuda(), W.t().contiguous().cuda()
    reps = [torch.full((n, N), float("nan"), dtype=torch.bfloat16, device="cuda") for _ in range(G)]
    for g in range(G):
        r0, r1 = M.row_block(n, G, g)
        ptrs = [reps[(g + k) % G].data_ptr() for k in range(G)]     # own replica first
        arr = (ctypes.c_void_p * G)(*ptrs)
        Xg = Xd[r0:r1]
        M.mps_xw_bf16_bcast(_p(Xg), r1 - r0, F, Xg.stride(0), _p(Wt), N, Wt.stride(0), arr, G,
                            r0, N, _stream())
    torch.cuda.synchronize()
    for k in range(G):
        assert torch.equal(reps[k].double().cpu(), ref), k


def test_xw_bcast_errors():
    import ctypes
    X = torch.zeros((10, 64), dtype=torch.bfloat16, device="cuda")
    Wt = torch.zeros((32, 64), dtype=torch.bfloat16, device="cuda")
    B = torch.zeros((10, 32), dtype=torch.bfloat16, device="cuda")
    arr = (ctypes.c_void_p * 17)(*([B.data_ptr()] * 17))
    with pytest.raises(M.MpsError):     # more than 16 destinations
        M.mps_xw_bf16_bcast(_p(X), 10, 64, 64, _p(Wt), 32, 64, arr, 17, 0, 32, _stream())
    arr1 = (ctypes.c_void_p * 1)(None)
    with pytest.raises(M.MpsError):     # NULL destination
        M.mps_xw_bf16_bcast(_p(X), 10, 64, 64, _p(Wt), 32, 64, arr1, 1, 0, 32, _stream())


def test_ipc_handle_offset():
    import ctypes
    t = torch.empty(1 << 20, dtype=torch.uint8, device="cuda")
    h, off = M.sharded.ipc_handle(t[4096:])
    assert len(h) == M.mps_ipc_handle_bytes() == 64
    h0, off0 = M.sharded.ipc_handle(t)
    assert off - off0 == 4096 and len(h0) == 64
    with pytest.raises(M.MpsError):     # a host pointer is not a device allocation
        buf = ctypes.create_string_buffer(64)
        o = ctypes.c_int64()
        M.mps_ipc_get_handle(ctypes.cast(buf, ctypes.c_void_p), buf, ctypes.byref(o))


_WORKER = r'''
import os, sys, json
sys.path.insert(0, sys.argv[1])
import torch, torch.distributed as dist
import oracle as O
import paper_conf_ispass_shangndk23_b200 as M
rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
torch.cuda.set_device(0)                      # both processes share the one GPU
dist.init_process_group("gloo")
n, F, N = 3001, 100, 128
g = torch.Generator(device="cpu").manual_seed(5)
X = torch.randint(-1, 2, (n, F), generator=g).to(torch.bfloat16)
W = torch.randint(-1, 2, (F, N), generator=g).to(torch.bfloat16)
ref = torch.from_numpy(O.xw_f64(X.float().numpy(), W.float().numpy()))
ldx = 104                                     # TMA row stride must be 16-B aligned
Xp = torch.zeros((n, ldx), dtype=torch.bfloat16); Xp[:, :F] = X
Wt = torch.zeros((N, ldx), dtype=torch.bfloat16); Wt[:, :F] = W.t()
rep = M.PeerReplicas(n, N, rank, world, "cuda:0")
rep.B.fill_(float("nan"))
torch.cuda.synchronize(); dist.barrier()
r0, r1 = M.row_block(n, world, rank)
B = M.xw_replicate(Xp.cuda()[r0:r1, :F], Wt.cuda()[:, :F], rep)
ok = bool(torch.equal(B.double().cpu(), ref))
dist.barrier()
rep.close()
print(json.dumps({"rank": rank, "ok": ok}))
dist.destroy_process_group()
'''


def test_xw_replicate_two_processes_ipc(tmp_path):
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    w = tmp_path / "worker.py"
    w.write_text(_WORKER)
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr", "127.0.0.1", "--master-port", str(port), str(w), ROOT]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    # the two ranks share stdout: their lines may interleave, so match the records
    oks = re.findall(r'\{"rank": (\d+), "ok": (true|false)\}', r.stdout)
    assert sorted(int(k) for k, _ in oks) == [0, 1] and all(v == "true" for _, v in oks), r.stdout
