"""NEXT-3 multi-GPU: one GCN aggregation layer A*(X*W) with the replication of B = X*W
pipelined against the sharded SpMM (ShardedGCNLayer: mps_xw_bf16_bcast per column
tile, mps_peer_signal / mps_peer_wait, mps_spmm_shard_p2p per tile).  Integer-valued X,
W and A: B is exact in bf16 and C must equal oracle O1 on the fp64 product bit-exactly.

Loopback on one GPU: G ranks' combinations on one stream, then per column tile every
rank's wait + SpMM in rank order on a second stream (the waits overlap the first)."""
import re

import numpy as np
import pytest
import torch

import graphgen as G
import oracle as O

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_ispass_shangndk23_b200 as M


@pytest.mark.parametrize("world", [1, 2, 3, 4])
@pytest.mark.parametrize("N,tile", [(64, 16), (128, 64), (96, 32)])
def test_sharded_gcn_layer_loopback(world, N, tile):
    rs = np.random.RandomState(world * 7 + N)
    n, F = 700, 72
    rl = rs.randint(0, 12, size=n).astype(np.int32)
    rl[rs.randint(n)] = 900
    g = G.random_csr(n, n, rl, 5)
    gen = torch.Generator().manual_seed(N)
    X = torch.randint(-1, 2, (n, F), generator=gen).to(torch.bfloat16)
    W = torch.randint(-1, 2, (F, N), generator=gen).to(torch.bfloat16)
    Bref = O.xw_f64(X.float().numpy(), W.float().numpy())     # |.| <= 72: exact in bf16
    ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, Bref, want_bound=False)
    Xd, Wt = X.cuda(), W.t().contiguous().cuda()
    Bs = [torch.full((n, N), float("nan"), dtype=torch.bfloat16, device="cuda")
          for _ in range(world)]
    sigs = [torch.zeros(int(M.mps_signal_bytes()), dtype=torch.uint8, device="cuda")
            for _ in range(world)]
    boxes = [torch.zeros(int(M.mps_shard_mailbox_bytes(N)), dtype=torch.uint8, device="cuda")
             for _ in range(world)]
    layers = []
    for r in range(world):
        peers = dict(replicas=[b.data_ptr() for b in Bs], signals=[t.data_ptr() for t in sigs],
                     mailboxes=[t.data_ptr() for t in boxes], B=Bs[r])
        layers.append(M.ShardedGCNLayer(g.row_ptr, g.col_idx, g.val, n, F, N, r, world, "cuda",
                                        tile_cols=tile, items_per_part=23, min_parts=1,
                                        peers=peers))
    s_xw, s_agg = torch.cuda.Stream(), torch.cuda.Stream()
    for step in range(3):                                     # epochs and slots reused
        for L_ in layers:
            L_.sh.C.fill_(float("nan"))
        torch.cuda.synchronize()
        for L_ in layers:
            r0, r1 = L_.r0, L_.r1
            L_.replicate(Xd[r0:r1], Wt, s_xw)
        for slot in range(len(layers[0].tiles)):
            for L_ in layers:
                L_.aggregate_tile(slot, s_agg)
        torch.cuda.synchronize()
        for r, L_ in enumerate(layers):
            assert torch.equal(Bs[r].double().cpu(), torch.from_numpy(Bref)), (step, r)
        C = np.concatenate([L_.sh.C[: L_.sh.rows].cpu().numpy() for L_ in layers])
        assert np.array_equal(C.astype(np.float64), ref), step


_WORKER = r'''
import os, sys, json
sys.path.insert(0, sys.argv[1])
import numpy as np, torch, torch.distributed as dist
import graphgen as G, oracle as O
import paper_conf_ispass_shangndk23_b200 as M
rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
torch.cuda.set_device(0)
dist.init_process_group("gloo")
n, F, N = 900, 64, 128
rs = np.random.RandomState(1)
rl = rs.randint(0, 10, size=n).astype(np.int32); rl[450] = 2000
g = G.random_csr(n, n, rl, 2)
gen = torch.Generator().manual_seed(9)
X = torch.randint(-1, 2, (n, F), generator=gen).to(torch.bfloat16)
W = torch.randint(-1, 2, (F, N), generator=gen).to(torch.bfloat16)
Bref = O.xw_f64(X.float().numpy(), W.float().numpy())
ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, Bref, want_bound=False)
layer = M.ShardedGCNLayer(g.row_ptr, g.col_idx, g.val, n, F, N, rank, world, "cuda:0",
                          tile_cols=32, items_per_part=31, min_parts=1)
r0, r1 = layer.r0, layer.r1
Xr, Wt = X.cuda()[r0:r1], W.t().contiguous().cuda()
ok = True
for step in range(3):
    torch.cuda.synchronize(); dist.barrier()
    C = layer(Xr, Wt); torch.cuda.synchronize(); dist.barrier()
    x0, x1 = int(layer.sh.X[rank]), int(layer.sh.X[rank + 1])
    ok = ok and np.array_equal(C.cpu().numpy().astype(np.float64), ref[x0:x1])
layer.close()
print(json.dumps({"rank": rank, "ok": bool(ok)}))
dist.destroy_process_group()
'''


def test_sharded_gcn_layer_two_processes_ipc(tmp_path):
    import os, socket, subprocess, sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    w = tmp_path / "worker.py"
    w.write_text(_WORKER)
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr", "127.0.0.1", "--master-port", str(port), str(w), root]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    # the two ranks share stdout: their lines may interleave, so match the records
    oks = re.findall(r'\{"rank": (\d+), "ok": (true|false)\}', r.stdout)
    assert sorted(int(k) for k, _ in oks) == [0, 1] and all(v == "true" for _, v in oks), r.stdout


_WORKER_B2B = r'''
import os, sys, json
sys.path.insert(0, sys.argv[1])
import numpy as np, torch, torch.distributed as dist
import graphgen as G, oracle as O
import paper_conf_ispass_shangndk23_b200 as M
rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
torch.cuda.set_device(0)
dist.init_process_group("gloo")
n, F, N = 1500, 64, 128
rs = np.random.RandomState(3)
rl = rs.randint(0, 10, size=n).astype(np.int32); rl[700] = 3000
g = G.random_csr(n, n, rl, 4)
W = torch.randint(-1, 2, (F, N), generator=torch.Generator().manual_seed(5)).to(torch.bfloat16)
Xs = [torch.randint(-1, 2, (n, F), generator=torch.Generator().manual_seed(10 + k)).to(torch.bfloat16)
      for k in range(5)]
layer = M.ShardedGCNLayer(g.row_ptr, g.col_idx, g.val, n, F, N, rank, world, "cuda:0",
                          tile_cols=32, items_per_part=31, min_parts=1)
r0, r1 = layer.r0, layer.r1
Wt = W.t().contiguous().cuda()
Xd = [X.cuda()[r0:r1].contiguous() for X in Xs]
s_xw, s_agg = torch.cuda.Stream(), torch.cuda.Stream()
outs = []
torch.cuda.synchronize(); dist.barrier()
for k in range(5):          # back to back: no synchronisation, no barrier between calls
    C = layer(Xd[k], Wt, s_xw=s_xw, s_agg=s_agg)
    with torch.cuda.stream(s_agg):
        outs.append(C.clone())
torch.cuda.synchronize(); dist.barrier()
ok = True
x0, x1 = int(layer.sh.X[rank]), int(layer.sh.X[rank + 1])
for k in range(5):
    Bref = O.xw_f64(Xs[k].float().numpy(), W.float().numpy())
    ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, Bref, want_bound=False)
    ok = ok and np.array_equal(outs[k].cpu().numpy().astype(np.float64), ref[x0:x1])
layer.close()
print(json.dumps({"rank": rank, "ok": bool(ok)}))
dist.destroy_process_group()
'''


def test_sharded_gcn_layer_back_to_back_calls(tmp_path):
    """a call must not overwrite a peer's B replica while that peer's SpMM of
    the previous call still gathers from it (consumed-acks in ShardedGCNLayer).  Five
    calls with a different X each, no synchronisation or barrier between them."""
    import os, socket, subprocess, sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    w = tmp_path / "worker_b2b.py"
    w.write_text(_WORKER_B2B)
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr", "127.0.0.1", "--master-port", str(port), str(w), root]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    oks = re.findall(r'\{"rank": (\d+), "ok": (true|false)\}', r.stdout)
    assert sorted(int(k) for k, _ in oks) == [0, 1] and all(v == "true" for _, v in oks), r.stdout


def _bf16_rne(a):
    """fp32 -> bf16 round-to-nearest-even (the kernels' __float2bfloat16_rn), as float64."""
    u = np.ascontiguousarray(a, np.float32).view(np.uint32).astype(np.uint64)
    u = (u + 0x7FFF + ((u >> 16) & 1)) & 0xFFFF0000
    return u.astype(np.uint32).view(np.float32).astype(np.float64)


@pytest.mark.parametrize("world", [1, 2, 3])
def test_sharded_gcn2_loopback(world):
    """out = A*(relu(A*(X*W1))*W2) with the bf16 roundings at the same three points as the
    kernels (B1, H, B2); integer inputs keep every fp32 sum exact -> bit-exact."""
    rs = np.random.RandomState(world)
    n, F, Hd, Cd = 600, 24, 32, 16
    rl = rs.randint(0, 9, size=n).astype(np.int32)
    rl[rs.randint(n)] = 400
    g = G.random_csr(n, n, rl, 11)
    gen = torch.Generator().manual_seed(world)
    X = torch.randint(-1, 2, (n, F), generator=gen).to(torch.bfloat16)
    W1 = torch.randint(-1, 2, (F, Hd), generator=gen).to(torch.bfloat16)
    W2 = torch.randint(-1, 2, (Hd, Cd), generator=gen).to(torch.bfloat16)
    B1 = _bf16_rne(O.xw_f64(X.float().numpy(), W1.float().numpy()))
    C1 = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B1, want_bound=False)
    Hh = _bf16_rne(np.maximum(C1, 0.0))
    B2 = _bf16_rne(O.xw_f64(Hh.astype(np.float32), W2.float().numpy()))
    ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B2, want_bound=False)

    def peers(N):
        Bs = [torch.empty((n, N), dtype=torch.bfloat16, device="cuda") for _ in range(world)]
        sg = [torch.zeros(int(M.mps_signal_bytes()), dtype=torch.uint8, device="cuda")
              for _ in range(world)]
        bx = [torch.zeros(int(M.mps_shard_mailbox_bytes(N)), dtype=torch.uint8, device="cuda")
              for _ in range(world)]
        keep.extend(Bs + sg + bx)
        return [dict(replicas=[b.data_ptr() for b in Bs], signals=[t.data_ptr() for t in sg],
                     mailboxes=[t.data_ptr() for t in bx], B=Bs[r]) for r in range(world)]
    keep = []
    p1, p2 = peers(Hd), peers(Cd)
    nets = [M.ShardedGCN2(g.row_ptr, g.col_idx, g.val, n, W1.cuda(), W2.cuda(), r, world,
                          "cuda", tile_cols=16, peers1=p1[r], peers2=p2[r], items_per_part=19,
                          min_parts=1) for r in range(world)]
    Xd = X.cuda()
    s_xw, s_agg = torch.cuda.Stream(), torch.cuda.Stream()
    for step in range(2):
        for net in nets:                                  # layer 1, loopback order
            net.l1.replicate(Xd[net.l1.r0:net.l1.r1], net.W1t, s_xw)
        for slot in range(len(nets[0].l1.tiles)):
            for net in nets:
                net.l1.aggregate_tile(slot, s_agg)
        Hs = [net.hidden(s_agg) for net in nets]
        s_xw.wait_stream(s_agg)
        for net, Hr in zip(nets, Hs):                     # layer 2
            net.l2.replicate(Hr, net.W2t, s_xw)
        for slot in range(len(nets[0].l2.tiles)):
            for net in nets:
                net.l2.aggregate_tile(slot, s_agg)
        torch.cuda.synchronize()
        out = np.concatenate([net.l2.sh.C[: net.l2.sh.rows].cpu().numpy() for net in nets])
        assert np.array_equal(out.astype(np.float64), ref), step
