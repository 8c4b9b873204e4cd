"""B200-native MergePath-SpMM (Shan et al., ISPASS 2023): C = A * B for an ultra-sparse
power-law CSR adjacency A and a dense, tall and thin B = X*W.

The compute lives in libmpspmm.so (hand-written CUDA for sm_100a behind the C ABI of
include/mpspmm.h).  This package is the thin Python binding: ``_lib`` mirrors the C
entry points one to one; ``api`` and ``sharded`` marshal torch tensors to them.
"""
from . import _lib
from ._lib import *  # noqa: F401,F403  (mps_* entry points, MpsError, constants)
from .api import (CSR, CapturedSpMM, OnlineStep, Schedule, mps_csr_host, partition, plan, spmm, spmm_host,  # noqa: F401
                  spmm_host_dense,
                  validate_csr, write_counts, write_stats, xw_bf16)
from .gcn import GCN2  # noqa: F401
from .sharded import (PeerReplicas, ShardedGCN2, ShardedGCNLayer, ShardedSpMM, exchange_tails, replicate_B, row_block,  # noqa: F401
                      shard_bounds, xw_replicate)

__all__ = ["GCN2", "CSR", "CapturedSpMM", "OnlineStep", "Schedule", "plan", "partition", "spmm", "spmm_host", "spmm_host_dense", "write_stats", "write_counts",
           "validate_csr", "xw_bf16", "ShardedSpMM", "shard_bounds", "exchange_tails", "replicate_B",
           "PeerReplicas", "xw_replicate", "row_block", "ShardedGCNLayer", "ShardedGCN2"] + list(_lib.EXPORTED)
