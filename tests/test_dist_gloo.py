"""Multi-process (world_size 2 and 4, gloo, CPU) test of the a6 sharding plumbing.

Every rank computes the shard bounds with the library's host entry point
(mps_shard_bounds), produces its local rows and tail vector (here with the oracle --
the device kernels need a GPU), exchanges the tails with the product's
`exchange_tails` collective, and settles the rows it owns by the owner rule in
ascending rank order.  Rank 0 gathers the row blocks and checks the assembled C
against the oracle bit-exactly (integer inputs)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import graphgen as G
import oracle as O


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _graph(seed):
    rl = np.ones(60, np.int32)
    rl[17] = 400                        # one long row spanning several shards
    rl[40:45] = 0
    g = G.random_csr(60, 50, rl, seed)
    return g


def _worker(rank, world, port, result_q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_ispass_shangndk23_b200.sharded import exchange_tails, shard_bounds
        ok = True
        for seed in (1, 2, 3):
            g = _graph(seed)
            K = 5
            B = G.dense_int(g.n, K, seed=seed)
            X, Y, T = shard_bounds(g.row_ptr, world)
            ox, oy, ot = O.shard(g.row_ptr, world)
            ok &= np.array_equal(X, ox) and np.array_equal(Y, oy) and np.array_equal(T, ot)
            C_local, tail = O.shard_local(g.row_ptr, g.col_idx, g.val, B, X, Y, rank)
            tails = exchange_tails(torch.from_numpy(tail.astype(np.float32)), world)
            tails = tails.view(world, K).numpy().astype(np.float64)
            for h in range(world):                       # ascending rank order
                r = int(T[h])
                if r < 0:
                    continue
                owner = max(gg for gg in range(world) if X[gg] <= r)
                if owner == rank:
                    C_local[r - X[rank]] += tails[h]
            # gather the row blocks on every rank (pad to the largest block)
            rows = int(X[rank + 1] - X[rank])
            maxr = int(max(X[i + 1] - X[i] for i in range(world)))
            buf = torch.zeros(maxr, K, dtype=torch.float64)
            buf[:rows] = torch.from_numpy(C_local)
            allb = [torch.zeros_like(buf) for _ in range(world)]
            dist.all_gather(allb, buf)
            C = np.concatenate([allb[i][: int(X[i + 1] - X[i])].numpy() for i in range(world)])
            ref = O.csr_spmm_f64(g.row_ptr, g.col_idx, g.val, B, want_bound=False)
            ok &= C.shape == ref.shape and np.array_equal(C, ref)
        result_q.put((rank, bool(ok)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4])
def test_gloo_shard_exchange(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    assert all(ok for _, ok in res), res
