"""a6 with the tail exchange over peer memory (mps_spmm_shard_p2p): the last CTA of the
kernel that finalises a rank's tail pushes it into the owner's mailbox and the owner's
last CTA pulls, in ascending rank order.  Integer inputs: every step's assembled C must
equal oracle O1 bit-exactly, in both fix-up modes, for several consecutive epochs (the
two inbox slots and the acknowledgements are exercised).

1. Loopback on one GPU: G ranks launched in rank order on one stream (a rank only waits
   for lower ranks, so rank order never blocks).
2. Two processes on one GPU with real CUDA IPC mailboxes (gloo process group).
"""
import ctypes
import os
import re
import socket
import subprocess
import sys

import numpy as np
import pytest
import torch

import graphgen as G
import oracle as O

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

if torch.cuda.is_available():
    import paper_conf_ispass_shangndk23_b200 as M


def graphs():
    rs = np.random.RandomState(0)
    out = []
    rl = np.ones(60, np.int32)
    rl[17] = 400                                   # one row spanning several shards
    rl[40:45] = 0
    out.append(G.random_csr(60, 50, rl, 1))
    rl = rs.randint(0, 30, size=500).astype(np.int32)
    rl[0], rl[250], rl[-1] = 3000, 2000, 3000      # evil rows at both ends and middle
    out.append(G.random_csr(500, 300, rl, 2))
    out.append(G.random_csr(3, 5, np.array([0, 2, 0], np.int32), 3))   # shards without items
    return out


@pytest.mark.parametrize("fixup", ["atomic", "carry"])
@pytest.mark.parametrize("world", [2, 3, 4, 8, 16])
@pytest.mark.parametrize("K", [12, 64, 200])
def test_p2p_tails_loopback(fixup, world, K):
    for gi, g in enumerate(graphs()):
        B = G.dense_int(g.n, K, seed=gi)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        Bt = torch.from_numpy(B).cuda()
        nb = int(M.mps_shard_mailbox_bytes(K))
        boxes = [torch.zeros(nb, dtype=torch.uint8, device="cuda") for _ in range(world)]
        ptrs = [b.data_ptr() for b in boxes]
        sh = [M.ShardedSpMM(g.row_ptr, g.col_idx, g.val, g.n, K, r, world, "cuda",
                            fixup=fixup, items_per_part=7, min_parts=1, tails="p2p",
                            mailbox_ptrs=ptrs) for r in range(world)]
        for step in range(4):
            for s in sh:
                s.C.fill_(float("nan"))
            outs = [s.local_p2p(Bt) for s in sh]      # rank order on one stream
            torch.cuda.synchronize()
            C = np.concatenate([o.cpu().numpy() for o in outs])
            assert np.array_equal(C.astype(np.float64), ref), (gi, step)
        # flags and acks: 0 (never used) or the last epoch, and the launch counters reset
        for r in range(world):
            words = boxes[r][:192].view(torch.int32).cpu().numpy()
            assert words[0] == 0
            assert set(words[16:16 + world].tolist()) <= {0, 4}
            assert set(words[32:32 + world].tolist()) <= {0, 4}


_WORKER = r'''
import os, sys, json
sys.path.insert(0, sys.argv[1])
import numpy as np, torch, torch.distributed as dist
import graphgen as G, oracle as O
import paper_conf_ispass_shangndk23_b200 as M
rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
torch.cuda.set_device(0)
dist.init_process_group("gloo")
rl = np.ones(80, np.int32); rl[30] = 5000; rl[31:35] = 0
g = G.random_csr(80, 70, rl, 9)
K = 64
B = G.dense_int(g.n, K, seed=4)
ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
ok = True
for fixup in ("atomic", "carry"):
    sh = M.ShardedSpMM(g.row_ptr, g.col_idx, g.val, g.n, K, rank, world, "cuda:0", fixup=fixup,
                       items_per_part=16, min_parts=1, tails="p2p")
    Bt = torch.from_numpy(B).cuda()
    for step in range(3):
        sh.C.fill_(float("nan")); torch.cuda.synchronize(); dist.barrier()
        C = sh(Bt); torch.cuda.synchronize(); dist.barrier()
        r0, r1 = int(sh.X[rank]), int(sh.X[rank + 1])
        ok = ok and np.array_equal(C.cpu().numpy().astype(np.float64), ref[r0:r1])
    sh.mail.close()
print(json.dumps({"rank": rank, "ok": bool(ok)}))
dist.destroy_process_group()
'''


def test_p2p_tails_two_processes_ipc(tmp_path):
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


@pytest.mark.parametrize("tails", ["nccl", "p2p"])
@pytest.mark.parametrize("fixup", ["atomic", "carry"])
def test_sharded_int64_loopback(tails, fixup):
    """NEXT-4 scale-out: sharding with 64-bit indices (mps_spmm_shard64), both exchanges."""
    world, K = 4, 40
    for gi, g in enumerate(graphs()):
        B = G.dense_int(g.n, K, seed=gi)
        ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
        Bt = torch.from_numpy(B).cuda()
        rp64 = g.row_ptr.astype(np.int64)
        ptrs = None
        if tails == "p2p":
            nb = int(M.mps_shard_mailbox_bytes(K))
            boxes = [torch.zeros(nb, dtype=torch.uint8, device="cuda") for _ in range(world)]
            ptrs = [b.data_ptr() for b in boxes]
        sh = [M.ShardedSpMM(rp64, g.col_idx, g.val, g.n, K, r, world, "cuda", fixup=fixup,
                            items_per_part=9, min_parts=1, tails=tails, mailbox_ptrs=ptrs)
              for r in range(world)]
        assert all(s.wide for s in sh)
        for step in range(2):
            if tails == "p2p":
                outs = [s.local_p2p(Bt) for s in sh]
            else:
                for s in sh:
                    s.local(Bt)
                allt = torch.cat([s.tail for s in sh])
                outs = [s.settle(allt) for s in sh]
            torch.cuda.synchronize()
            C = np.concatenate([o.cpu().numpy() for o in outs])
            assert np.array_equal(C.astype(np.float64), ref), (gi, step)
