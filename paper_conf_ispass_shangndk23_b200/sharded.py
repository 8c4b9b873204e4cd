"""a6: merge-path sharding of C = A*B over G GPUs (north-star stage 4; not in the paper).

One process per GPU (torch.distributed, NCCL over NVLink/NVSwitch).  The merge path of
A is cut into G equal slices of rows + non-zeros (the paper's Alg. 1 applied with G
"threads"), so every GPU gets the same item count and, by the byte balance of
DESIGN.md, the same memory traffic.  B is replicated (read-only); GPU g owns C rows
[X_g, X_{g+1}).  The only exchange is the tail record of a row cut by a slice edge:
one all-gather of G x K floats, after which each owner adds the tails of its row in
ascending rank order (deterministic).
"""
from __future__ import annotations

import ctypes

import numpy as np
import torch
import torch.distributed as dist

from . import _lib as L
from .api import CSR, _p, _stream, _fix, _dtype_code, _ws


def shard_bounds(row_ptr_host: np.ndarray, world: int):
    """Host closed form (mps_shard_bounds / mps_shard_bounds64 for an int64 row_ptr):
    X (int32[world+1]), Y (row_ptr's index type, [world+1]) and tail rows."""
    wide = np.asarray(row_ptr_host).dtype == np.int64
    it = np.int64 if wide else np.int32
    rp = np.ascontiguousarray(row_ptr_host, it)
    m, nnz = rp.shape[0] - 1, int(rp[-1])
    X = np.zeros(world + 1, np.int32)
    Y = np.zeros(world + 1, it)
    T = np.zeros(world, np.int32)
    (L.mps_shard_bounds64 if wide else L.mps_shard_bounds)(_p(rp), m, nnz, world, _p(X), _p(Y),
                                                           _p(T))
    return X, Y, T


def exchange_tails(tail: torch.Tensor, world: int, group=None) -> torch.Tensor:
    """All-gather every rank's tail vector (K floats) -> (world*K,) rank-major.

    This is the path's only collective (NCCL on GPUs, gloo in the CPU tests)."""
    out = torch.empty(world * tail.numel(), dtype=tail.dtype, device=tail.device)
    if world == 1:
        out.copy_(tail.reshape(-1))
        return out
    if tail.is_cuda and dist.get_backend(group) == "gloo":
        # gloo has no device all-gather: stage through host memory (test/debug runs only;
        # production multi-GPU runs use NCCL over NVLink)
        host = torch.empty(world * tail.numel(), dtype=tail.dtype)
        dist.all_gather_into_tensor(host, tail.reshape(-1).cpu(), group=group)
        out.copy_(host)
        return out
    dist.all_gather_into_tensor(out, tail.reshape(-1).contiguous(), group=group)
    return out


def replicate_B(B_rows: torch.Tensor, n: int, world: int, group=None) -> torch.Tensor:
    """Replicate B over the ranks (north-star stage 4: "replicates B over NVLink").

    Rank g holds rows [g*ceil(n/G), (g+1)*ceil(n/G)) of B (the last shard padded); one
    all_gather_into_tensor (NCCL over NVLink/NVSwitch) assembles the full n x K B on
    every rank.  It runs once per B (offline setting), outside the SpMM step."""
    per = -(-n // world)
    K = B_rows.shape[1]
    shard = torch.zeros((per, K), dtype=B_rows.dtype, device=B_rows.device)
    shard[: B_rows.shape[0]] = B_rows
    full = torch.empty((per * world, K), dtype=B_rows.dtype, device=B_rows.device)
    if world == 1:
        full.copy_(shard)
    elif shard.is_cuda and dist.get_backend(group) == "gloo":   # test runs: host staging
        host = torch.empty(full.shape, dtype=full.dtype)
        dist.all_gather_into_tensor(host, shard.cpu(), group=group)
        full.copy_(host)
    else:
        dist.all_gather_into_tensor(full, shard, group=group)
    return full[:n]


def _agree(ok: bool, device, group=None) -> bool:
    """One all_reduce(MIN) of a success flag: True only if every rank succeeded."""
    dev = device if dist.get_backend(group) == "nccl" else "cpu"
    t = torch.tensor([1 if ok else 0], dtype=torch.int32, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MIN, group=group)
    return bool(int(t[0]) == 1)


def _open_peers(buf: torch.Tensor, rank: int, world: int, group=None):
    """All ranks' device pointers to their `buf` (CUDA IPC), indexed by rank, plus the
    bases this process opened (to close later).  Collective-safe: every rank takes part
    in the same collectives whatever fails locally, and the ranks agree on success
    before returning, so the call returns on all ranks or raises on all ranks."""
    err = None
    try:
        mine = ipc_handle(buf)
    except Exception as e:
        mine, err = None, e
    allh = [None] * world
    dist.all_gather_object(allh, mine, group=group)
    ptrs, opened = [], []
    if err is None and all(h is not None for h in allh):
        try:
            for g in range(world):
                if g == rank:
                    ptrs.append(buf.data_ptr())
                    continue
                h, off = allh[g]
                base = ctypes.c_void_p()
                L.mps_ipc_open_handle(ctypes.create_string_buffer(h, len(h)), ctypes.byref(base))
                opened.append(base.value)
                ptrs.append(base.value + off)
        except Exception as e:
            err = e
    else:
        err = err or RuntimeError("a peer could not export its IPC handle")
    if not _agree(err is None, buf.device, group):
        for b in opened:
            L.mps_ipc_close_handle(ctypes.c_void_p(b))
        raise RuntimeError("peer mapping failed on some rank (this rank: %s)" % (err,))
    return ptrs, opened


class Mailboxes:
    """The a6 peer-memory tail exchange's mailboxes (mps_shard_mailbox_bytes each): this
    rank's own, zeroed, and every peer's mapped through CUDA IPC.  ``ptrs`` is indexed
    by rank.  For loopback use in one process pass ``ptrs`` of local buffers instead."""

    def __init__(self, K: int, rank: int, world: int, device, group=None, ptrs=None):
        self.buf = torch.zeros(int(L.mps_shard_mailbox_bytes(K)), dtype=torch.uint8,
                               device=device)
        self._opened = []
        if ptrs is not None:
            self.ptrs = list(ptrs)
        else:
            torch.cuda.synchronize(device)
            self.ptrs, self._opened = _open_peers(self.buf, rank, world, group)
            dist.barrier(group=group)        # every mailbox zeroed before any push

    def close(self):
        for b in self._opened:
            L.mps_ipc_close_handle(ctypes.c_void_p(b))
        self._opened = []


class ShardedSpMM:
    """Rank-local state of a merge-path sharded SpMM.

    row_ptr/col_idx/val: the global CSR on the host (numpy); every rank computes the
    same bounds, uploads the full row_ptr and only its own [Y_g, Y_{g+1}) slice.
    tails="nccl": the tail vectors are exchanged by one all-gather (exchange_tails) and
    settled by mps_apply_tails; tails="p2p": the kernel that finalises the tail pushes it
    into the owner's mailbox over peer memory and pulls the tails owned by this rank
    (mps_spmm_shard_p2p) -- no collective, no extra launch."""

    def __init__(self, row_ptr, col_idx, val, n_cols, K, rank, world, device,
                 b_dtype=torch.float32, fixup="atomic", items_per_part=0, min_parts=0,
                 group=None, tails="nccl", mailbox_ptrs=None):
        self.rank, self.world, self.group, self.K = rank, world, group, K
        self.device = torch.device(device)
        self.fixup, self.ipp, self.minp = fixup, items_per_part, min_parts
        self.X, self.Y, self.T = shard_bounds(row_ptr, world)
        y0, y1 = int(self.Y[rank]), int(self.Y[rank + 1])
        t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).to(self.device)
        self.row_ptr = t(row_ptr)
        self.col = t(col_idx[y0:y1])
        self.val = t(val[y0:y1])
        self.m, self.n, self.nnz = len(row_ptr) - 1, int(n_cols), int(row_ptr[-1])
        self.row0 = int(self.X[rank])
        self.rows = int(self.X[rank + 1]) - self.row0
        self.C = torch.empty((max(self.rows, 1), K), dtype=torch.float32, device=self.device)
        self.tail = torch.zeros(K, dtype=torch.float32, device=self.device)
        self.wide = self.row_ptr.dtype == torch.int64     # NEXT-4: 64-bit indices
        cls = L.mps_csr64 if self.wide else L.mps_csr
        self.a = cls(self.m, self.n, self.nnz, _p(self.row_ptr), _p(self.col), _p(self.val))
        dt = L.MPS_DT_BF16 if b_dtype == torch.bfloat16 else L.MPS_DT_F32
        nb = ctypes.c_size_t()
        (L.mps_spmm_shard64_workspace_bytes if self.wide else L.mps_spmm_shard_workspace_bytes)(
            ctypes.byref(self.a), K, dt, _p(self.X), rank, world, items_per_part, min_parts,
            _fix(fixup), ctypes.byref(nb))
        self.ws = _ws(nb.value, self.device)
        self.tails = "nccl"
        self.epoch = 0
        self.mail = None
        if tails == "p2p":
            self.enable_p2p(mailbox_ptrs)

    def enable_p2p(self, mailbox_ptrs=None):
        """Switch the tail exchange to peer memory: map every rank's mailbox (CUDA IPC;
        collective over the group, succeeds or raises on every rank together)."""
        self.tails = "p2p"
        if self.world > 1 and self.mail is None:
            self.mail = Mailboxes(self.K, self.rank, self.world, self.device, self.group,
                                  ptrs=mailbox_ptrs)
            self._mp = (ctypes.c_void_p * self.world)(*self.mail.ptrs)

    def local_p2p(self, B: torch.Tensor, stream=None, c0: int = 0, kt: int | None = None):
        """One step with the peer-memory tail exchange: afterwards this rank's C rows are
        final once every rank's launch of the same epoch has run.  c0/kt: only columns
        [c0, c0+kt) of B and C (a column tile; every rank must call the same sequence)."""
        dt = _dtype_code(B)
        kt = self.K - c0 if kt is None else kt
        self.epoch += 1
        Bs = B[:, c0:c0 + kt]
        Cp = self.C[:, c0:] if self.rows > 0 else None
        if self.mail is None:             # one rank: no tails to exchange
            assert self.world == 1
            args = (ctypes.byref(self.a), _p(Bs), dt, B.stride(0), kt, _p(self.X), _p(self.Y),
                    _p(self.T), 0, 1, self.ipp, self.minp, _p(Cp), self.C.stride(0),
                    _p(self.tail[c0:]), _fix(self.fixup))
            if self.wide:
                L.mps_spmm_shard64(*args, None, 0, _p(self.ws), self.ws.numel(), _stream(stream))
            else:
                L.mps_spmm_shard(*args, _p(self.ws), self.ws.numel(), _stream(stream))
            return self.C[: self.rows]
        f = L.mps_spmm_shard64 if self.wide else L.mps_spmm_shard_p2p
        f(ctypes.byref(self.a), _p(Bs), dt, B.stride(0), kt, _p(self.X), _p(self.Y),
          _p(self.T), self.rank, self.world, self.ipp, self.minp, _p(Cp), self.C.stride(0),
          _p(self.tail[c0:]), _fix(self.fixup), self._mp, self.epoch, _p(self.ws),
          self.ws.numel(), _stream(stream))
        return self.C[: self.rows]

    def local(self, B: torch.Tensor, stream=None):
        """a2-a4 on this rank's slice: C rows [X_g, X_{g+1}) and the tail vector."""
        dt = _dtype_code(B)
        args = (ctypes.byref(self.a), _p(B), dt, B.stride(0), self.K, _p(self.X), _p(self.Y),
                _p(self.T), self.rank, self.world, self.ipp, self.minp,
                _p(self.C) if self.rows > 0 else None, self.C.stride(0), _p(self.tail),
                _fix(self.fixup))
        if self.wide:
            L.mps_spmm_shard64(*args, None, 0, _p(self.ws), self.ws.numel(), _stream(stream))
        else:
            L.mps_spmm_shard(*args, _p(self.ws), self.ws.numel(), _stream(stream))
        return self.C[: self.rows], self.tail

    def settle(self, tails_all: torch.Tensor, stream=None):
        """Add the gathered tails owned by this rank (ascending rank order)."""
        L.mps_apply_tails(_p(tails_all), _p(self.X), _p(self.T), self.world, self.rank, self.K,
                          _p(self.C) if self.rows > 0 else None, self.C.stride(0),
                          _stream(stream))
        return self.C[: self.rows]

    def __call__(self, B: torch.Tensor):
        if self.mail is not None:
            return self.local_p2p(B)
        self.local(B)
        tails = exchange_tails(self.tail, self.world, self.group)
        return self.settle(tails)


# --------------------------------------------------------------------------------
# NEXT-3 multi-GPU: the combination B = X*W fused with the replication of B
# --------------------------------------------------------------------------------
def ipc_handle(t: torch.Tensor):
    """(handle bytes, byte offset) naming t's device memory for a peer process."""
    h = ctypes.create_string_buffer(int(L.mps_ipc_handle_bytes()))
    off = ctypes.c_int64()
    L.mps_ipc_get_handle(_p(t), h, ctypes.byref(off))
    return h.raw, off.value


class PeerReplicas:
    """One B replica per rank, every rank holding device pointers to all of them.

    Each rank allocates its own replica (n x N bf16); the CUDA IPC handles are exchanged
    with an all_gather_object over the process group and the peers' replicas are mapped
    into this process (peer access over NVLink/NVSwitch).  ``ptrs[0]`` is this rank's own
    replica, followed by the other ranks' in rank order after it (rank+1, rank+2, ...)."""

    def __init__(self, n: int, N: int, rank: int, world: int, device, group=None):
        self.n, self.N, self.rank, self.world = n, N, rank, world
        self.B = torch.empty((n, N), dtype=torch.bfloat16, device=device)
        self._opened = []
        mine = ipc_handle(self.B) if world > 1 else (b"", 0)
        allh = [None] * world
        if world > 1:
            dist.all_gather_object(allh, mine, group=group)
        ptrs = [self.B.data_ptr()]
        for k in range(1, world):
            g = (rank + k) % world
            h, off = allh[g]
            base = ctypes.c_void_p()
            L.mps_ipc_open_handle(ctypes.create_string_buffer(h, len(h)), ctypes.byref(base))
            self._opened.append(base.value)
            ptrs.append(base.value + off)
        self.ptrs = ptrs

    def close(self):
        for b in self._opened:
            L.mps_ipc_close_handle(ctypes.c_void_p(b))
        self._opened = []


def row_block(n: int, world: int, rank: int):
    """Rows [r0, r1) of B this rank computes: ceil(n/G) per rank, the last one short."""
    per = -(-n // world)
    r0 = min(n, rank * per)
    return r0, min(n, r0 + per)


def xw_replicate(X_rows: torch.Tensor, Wt: torch.Tensor, rep: PeerReplicas, stream=None,
                 group=None, sync=True):
    """B = X*W on this rank's row block, written by ONE kernel (mps_xw_bf16_bcast) into
    every rank's replica.  With sync=True the stream is synchronised and the ranks meet at
    a barrier, after which every replica holds the whole B."""
    r0, r1 = row_block(rep.n, rep.world, rep.rank)
    assert X_rows.shape[0] == r1 - r0 and X_rows.dtype == torch.bfloat16
    assert Wt.shape[0] == rep.N and Wt.shape[1] == X_rows.shape[1]
    arr = (ctypes.c_void_p * len(rep.ptrs))(*rep.ptrs)
    L.mps_xw_bf16_bcast(_p(X_rows), r1 - r0, X_rows.shape[1], X_rows.stride(0), _p(Wt), rep.N,
                        Wt.stride(0), arr, len(rep.ptrs), r0, rep.B.stride(0), _stream(stream))
    if sync:
        (torch.cuda.current_stream() if stream is None else stream).synchronize()
        if rep.world > 1:
            dist.barrier(group=group)
    return rep.B


class ShardedGCNLayer:
    """One GCN aggregation layer A*(X*W) on G GPUs with the replication of B = X*W
    pipelined against the SpMM (NEXT-3, multi-GPU).

    Rank g holds the merge-path shard g of A and the rows [X_g, X_{g+1}) of X -- the
    rows of C it owns, so one layer's output is the next layer's input without moving.  B is
    produced in column tiles of ``tile_cols`` columns; for tile c:
      stream ``s_xw``:  mps_xw_bf16_bcast writes this rank's rows of B[:, tile c] into
                        every rank's replica (peer HBM), then mps_peer_signal(slot c);
      stream ``s_agg``: mps_peer_wait(slot c) -- every rank's rows of tile c arrived --
                        then the sharded SpMM of tile c with the peer-memory tail exchange.
    The SpMM of tile c therefore overlaps the GEMM + NVLink transfer of tile c+1.
    Output: this rank's C rows (fp32, pre-activation).  ``peers``: for loopback use in
    one process, dict(replicas=[ptr per rank], signals=[ptr per rank],
    mailboxes=[ptr per rank]); otherwise CUDA IPC over the process group."""

    CONSUMED = 32     # first signal slot of the consumed-acks

    def __init__(self, row_ptr, col_idx, val, n, F, N, rank, world, device, tile_cols=64,
                 fixup="atomic", items_per_part=0, min_parts=0, group=None, peers=None):
        assert N % 16 == 0 and tile_cols % 16 == 0
        self.n, self.F, self.N, self.rank, self.world = n, F, N, rank, world
        self.device = torch.device(device)
        self.tile = min(tile_cols, N)
        self.tiles = [(c, min(self.tile, N - c)) for c in range(0, N, self.tile)]
        # signal slots: [0, 32) tile t produced (replicated) for an epoch, [32, 64) tile t
        # consumed (this epoch's SpMM of tile t finished reading every replica)
        assert len(self.tiles) <= self.CONSUMED
        self.sh = ShardedSpMM(row_ptr, col_idx, val, n, N, rank, world, device,
                              b_dtype=torch.bfloat16, fixup=fixup, items_per_part=items_per_part,
                              min_parts=min_parts, group=group, tails="p2p",
                              mailbox_ptrs=None if peers is None else peers["mailboxes"])
        self.B = torch.empty((n, N), dtype=torch.bfloat16, device=self.device)
        self.sig = torch.zeros(int(L.mps_signal_bytes()), dtype=torch.uint8, device=self.device)
        self._opened = []
        if peers is not None:
            rep_ptrs, sig_ptrs = list(peers["replicas"]), list(peers["signals"])
            self.B = peers["B"] if "B" in peers else self.B
        else:
            torch.cuda.synchronize(self.device)
            rep_ptrs, o1 = _open_peers(self.B, rank, world, group)
            sig_ptrs, o2 = _open_peers(self.sig, rank, world, group)
            self._opened = o1 + o2
            dist.barrier(group=group)
        # destinations for the combination: own replica first, then the others
        self._dst = [rep_ptrs[(rank + k) % world] for k in range(world)]
        self._sig = (ctypes.c_void_p * world)(*sig_ptrs)
        self._mysig = sig_ptrs[rank]
        self.epoch = 0
        # the rows of X this rank combines are the rows of C it owns (merge-path shard
        # rows), so a layer's output rows feed the next layer's combination in place
        self.r0, self.r1 = int(self.sh.X[rank]), int(self.sh.X[rank + 1])

    def replicate(self, X_rows: torch.Tensor, Wt: torch.Tensor, stream):
        """Enqueue B = X*W tile by tile into every replica, each tile followed by a signal.
        Tile t of this epoch overwrites every rank's replica only after every rank has
        acknowledged that its SpMM of tile t of the previous epoch is done (consumed-ack
        slot 32 + t), so back-to-back calls never overwrite B under a peer's gathers."""
        self.epoch += 1
        s = _stream(stream)
        for slot, (c0, kt) in enumerate(self.tiles):
            if self.epoch > 1:
                L.mps_peer_wait(ctypes.c_void_p(self._mysig), self.world, self.CONSUMED + slot,
                                self.epoch - 1, s)
            dst = (ctypes.c_void_p * self.world)(*[p + 2 * c0 for p in self._dst])
            Wc = Wt[c0:c0 + kt]
            L.mps_xw_bf16_bcast(_p(X_rows), self.r1 - self.r0, X_rows.shape[1], X_rows.stride(0),
                                _p(Wc), kt, Wt.stride(0), dst, self.world, self.r0, self.N, s)
            L.mps_peer_signal(self._sig, self.world, self.rank, slot, self.epoch, s)

    def aggregate_tile(self, slot: int, stream):
        """Enqueue: wait for tile `slot` from every rank, then its sharded SpMM."""
        c0, kt = self.tiles[slot]
        L.mps_peer_wait(ctypes.c_void_p(self._mysig), self.world, slot, self.epoch,
                        _stream(stream))
        out = self.sh.local_p2p(self.B, stream=stream, c0=c0, kt=kt)
        # consumed-ack: this rank no longer reads tile `slot` of its replica this epoch
        L.mps_peer_signal(self._sig, self.world, self.rank, self.CONSUMED + slot, self.epoch,
                          _stream(stream))
        return out

    def __call__(self, X_rows: torch.Tensor, Wt: torch.Tensor, s_xw=None, s_agg=None):
        s_xw = s_xw or torch.cuda.Stream(self.device)
        s_agg = s_agg or torch.cuda.current_stream(self.device)
        s_xw.wait_stream(torch.cuda.current_stream(self.device))
        self.replicate(X_rows, Wt, s_xw)
        for slot in range(len(self.tiles)):
            out = self.aggregate_tile(slot, s_agg)
        return out

    def close(self):
        for b in self._opened:
            L.mps_ipc_close_handle(ctypes.c_void_p(b))
        self._opened = []
        if self.sh.mail is not None:
            self.sh.mail.close()


class ShardedGCN2:
    """2-layer GCN inference  out = A*(relu(A*(X*W1))*W2)  on G GPUs (NEXT-3): two
    ShardedGCNLayer, the hidden rows never leave their rank; between the layers one
    library kernel applies the ReLU and converts to bf16 (mps_relu_to_bf16).  X_rows:
    this rank's rows [X_g, X_{g+1}) of X (bf16); W1: F x H, W2: H x C (torch, any dtype).
    Returns this rank's output rows (fp32)."""

    def __init__(self, row_ptr, col_idx, val, n, W1, W2, rank, world, device, tile_cols=64,
                 group=None, peers1=None, peers2=None, **kw):
        F, H = W1.shape
        C = W2.shape[1]
        self.W1t = W1.t().contiguous().to(device=device, dtype=torch.bfloat16)
        self.W2t = W2.t().contiguous().to(device=device, dtype=torch.bfloat16)
        self.l1 = ShardedGCNLayer(row_ptr, col_idx, val, n, F, H, rank, world, device,
                                  tile_cols=tile_cols, group=group, peers=peers1, **kw)
        self.l2 = ShardedGCNLayer(row_ptr, col_idx, val, n, H, C, rank, world, device,
                                  tile_cols=tile_cols, group=group, peers=peers2, **kw)
        rows = max(self.l1.r1 - self.l1.r0, 1)
        self.Hb = torch.empty((rows, H), dtype=torch.bfloat16, device=device)

    def hidden(self, stream=None):
        """relu(layer-1 rows) -> bf16, the next combination's input (one library kernel)."""
        rows = self.l1.r1 - self.l1.r0
        C1 = self.l1.sh.C
        L.mps_relu_to_bf16(_p(C1) if rows else None, rows, C1.shape[1], C1.stride(0),
                           _p(self.Hb) if rows else None, self.Hb.stride(0), _stream(stream))
        return self.Hb[:rows]

    def __call__(self, X_rows, s_xw=None, s_agg=None):
        s_agg = s_agg or torch.cuda.current_stream()
        self.l1(X_rows, self.W1t, s_xw=s_xw, s_agg=s_agg)
        H = self.hidden(s_agg)
        return self.l2(H, self.W2t, s_xw=s_xw, s_agg=s_agg)

    def close(self):
        self.l1.close()
        self.l2.close()
