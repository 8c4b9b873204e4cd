"""ctypes binding of libmpspmm.so -- one Python function per C-ABI entry point of
include/mpspmm.h, same names, argument marshalling only (every step of the path runs in
the library's CUDA kernels).  Importing this module loads the in-tree library and fails
loudly if it is missing and cannot be built: there is no CPU fallback."""
from __future__ import annotations

import ctypes
import os

HERE = os.path.dirname(os.path.abspath(__file__))
# MPS_LIB: load another build of the same library (A/B experiments on one GPU box)
LIB_PATH = os.environ.get("MPS_LIB") or os.path.join(HERE, "libmpspmm.so")

MPS_OK, MPS_ERR_INVALID, MPS_ERR_UNSUPPORTED, MPS_ERR_CUDA, MPS_ERR_WORKSPACE, MPS_ERR_COMM = range(6)
MPS_FIXUP_AUTO, MPS_FIXUP_ATOMIC, MPS_FIXUP_CARRY = 0, 1, 2
MPS_DT_F32, MPS_DT_BF16 = 0, 1
MPS_EPI_NONE, MPS_EPI_RELU = 0, 1
MPS_PATH_PARTITION_SEGMENTS, MPS_PATH_SMALL_FUSED = 0, 1

_i64, _i32, _p, _sz = ctypes.c_int64, ctypes.c_int32, ctypes.c_void_p, ctypes.c_size_t


class mps_csr(ctypes.Structure):
    _fields_ = [("m", _i64), ("n", _i64), ("nnz", _i64), ("row_ptr", _p), ("col_idx", _p),
                ("val", _p)]


class mps_csr64(ctypes.Structure):
    """NEXT-4: int64 row_ptr (m + nnz >= 2^31); col_idx stays int32."""
    _fields_ = [("m", _i64), ("n", _i64), ("nnz", _i64), ("row_ptr", _p), ("col_idx", _p),
                ("val", _p)]


class MpsError(RuntimeError):
    def __init__(self, status, fn, detail):
        super().__init__("%s -> %s: %s" % (fn, _STATUS.get(status, status), detail))
        self.status = status


_STATUS = {0: "MPS_OK", 1: "MPS_ERR_INVALID", 2: "MPS_ERR_UNSUPPORTED", 3: "MPS_ERR_CUDA",
           4: "MPS_ERR_WORKSPACE", 5: "MPS_ERR_COMM"}

# name -> argtypes (restype mps_status unless listed in _RESTYPES)
_SIGS = {
    "mps_abi_version": [],
    "mps_status_string": [_i32],
    "mps_last_error": [],
    "mps_plan": [_i64, _i64, _i32, _i32, _i64, _i64, _p, _p],
    "mps_partition": [_p, _i64, _i64, _i64, _i64, _i64, _i64, _p, _p, _p],
    "mps_partition_split": [_p, _i64, _i64, _i64, _i64, _p, _p, _p, _i64, _i32, _p],
    "mps_spmm_workspace_bytes": [_p, _i32, _i32, _i64, _i32, _p],
    "mps_spmm": [_p, _p, _i32, _i64, _i32, _p, _i64, _p, _p, _i64, _i32, _p, _sz, _p],
    "mps_spmm_ex": [_p, _p, _i32, _i64, _i32, _p, _i64, _p, _p, _i64, _i32, _i32, _p, _p, _sz, _p],
    "mps_spmm_write_counts": [_p, _p, _i32, _i64, _i32, _p, _i64, _p, _p, _i64, _i32, _p, _p,
                              _sz, _p],
    "mps_spmm_online_path": [_p, _p, _i32, _i64, _i32, _p, _i64, _i64, _i64, _i32, _p],
    "mps_spmm_online_ex": [_p, _p, _i32, _i64, _i32, _p, _i64, _i64, _i64, _i32, _i32, _p, _sz,
                           _p],
    "mps_zero_split_rows": [_p, _p, _p, _i64, _p, _i64, _i32, _p],
    "mps_spmm_segments": [_p, _p, _i32, _i64, _i32, _p, _i64, _p, _p, _i64, _i32, _p, _sz, _p],
    "mps_hot_rows_workspace_bytes": [_i64, _p],
    "mps_hot_budget_rows": [_p, _i32, _i32, _p],
    "mps_hot_rows": [_p, _i64, _p, _p, _sz, _p],
    "mps_spmm_segments_hot": [_p, _p, _i32, _i64, _i32, _p, _i64, _p, _p, _i64, _i32, _p, _p, _sz,
                              _p],
    "mps_spmm_online_workspace_bytes": [_p, _i32, _i32, _i64, _i64, _i32, _p],
    "mps_spmm_online": [_p, _p, _i32, _i64, _i32, _p, _i64, _i64, _i64, _i32, _p, _sz, _p],
    "mps_spmm_host_workspace_bytes": [_p, _i32, _i32, _i64, _i64, _i64, _i64, _i32, _p],
    "mps_spmm_host": [_p, _p, _i32, _i64, _i32, _p, _i64, _i64, _i64, _i32, _p, _sz, _p],
    "mps_write_stats": [_p, _p, _p, _i64, _p, _p],
    "mps_spmm_host_dense_workspace_bytes": [_p, _i32, _i32, _i64, _i64, _i64, _i64, _i32, _p],
    "mps_spmm_host_dense": [_p, _p, _i32, _i64, _i32, _p, _i64, _i64, _i64, _i32, _p, _sz, _p],
    "mps_xw_bf16": [_p, _i64, _i64, _i64, _p, _i32, _i64, _p, _i64, _p],
    "mps_shard_bounds": [_p, _i64, _i64, _i32, _p, _p, _p],
    "mps_spmm_shard_workspace_bytes": [_p, _i32, _i32, _p, _i32, _i32, _i64, _i64, _i32, _p],
    "mps_spmm_shard": [_p, _p, _i32, _i64, _i32, _p, _p, _p, _i32, _i32, _i64, _i64, _p, _i64,
                       _p, _i32, _p, _sz, _p],
    "mps_apply_tails": [_p, _p, _p, _i32, _i32, _i32, _p, _i64, _p],
    "mps_validate_csr": [_p, _p, _p],
    "mps_xw_bf16_bcast": [_p, _i64, _i64, _i64, _p, _i32, _i64, _p, _i32, _i64, _i64, _p],
    "mps_ipc_handle_bytes": [],
    "mps_signal_bytes": [],
    "mps_relu_to_bf16": [_p, _i64, _i32, _i64, _p, _i64, _p],
    "mps_peer_signal": [_p, _i32, _i32, _i32, ctypes.c_uint32, _p],
    "mps_peer_wait": [_p, _i32, _i32, ctypes.c_uint32, _p],
    "mps_ipc_get_handle": [_p, _p, _p],
    "mps_ipc_open_handle": [_p, _p],
    "mps_ipc_close_handle": [_p],
    "mps_shard_mailbox_bytes": [_i32],
    "mps_spmm_shard_p2p": [_p, _p, _i32, _i64, _i32, _p, _p, _p, _i32, _i32, _i64, _i64, _p,
                           _i64, _p, _i32, _p, ctypes.c_uint32, _p, _sz, _p],
    "mps_plan64": [_i64, _i64, _i32, _i32, _i64, _i64, _p, _p],
    "mps_partition64": [_p, _i64, _i64, _i64, _i64, _i64, _i64, _p, _p, _p],
    "mps_spmm64_workspace_bytes": [_p, _i32, _i32, _i64, _i32, _p],
    "mps_spmm64": [_p, _p, _i32, _i64, _i32, _p, _i64, _p, _p, _i64, _i32, _i32, _p, _sz, _p],
    "mps_spmm64_online_workspace_bytes": [_p, _i32, _i32, _i64, _i64, _i32, _p],
    "mps_spmm64_online": [_p, _p, _i32, _i64, _i32, _p, _i64, _i64, _i64, _i32, _i32, _p, _sz,
                          _p],
    "mps_write_stats64": [_p, _p, _p, _i64, _p, _p],
    "mps_shard_bounds64": [_p, _i64, _i64, _i32, _p, _p, _p],
    "mps_spmm_shard64_workspace_bytes": [_p, _i32, _i32, _p, _i32, _i32, _i64, _i64, _i32, _p],
    "mps_spmm_shard64": [_p, _p, _i32, _i64, _i32, _p, _p, _p, _i32, _i32, _i64, _i64, _p,
                         _i64, _p, _i32, _p, ctypes.c_uint32, _p, _sz, _p],
    "mps_validate_csr64": [_p, _p, _p],
}
_RESTYPES = {"mps_abi_version": ctypes.c_int, "mps_status_string": ctypes.c_char_p,
             "mps_last_error": ctypes.c_char_p, "mps_ipc_handle_bytes": ctypes.c_size_t,
             "mps_shard_mailbox_bytes": ctypes.c_size_t, "mps_signal_bytes": ctypes.c_size_t}


def _load():
    if not os.path.exists(LIB_PATH):
        try:
            from . import _build
            _build.build()
        except Exception as e:  # no silent fallback: the CUDA path is the product
            raise ImportError("libmpspmm.so is missing and could not be built: %s" % e) from e
    lib = ctypes.CDLL(LIB_PATH)
    if not all(hasattr(lib, name) for name in _SIGS) and "MPS_LIB" not in os.environ:
        # a stale in-tree build that predates an entry point: rebuild it once, reload
        import _ctypes
        from . import _build
        _ctypes.dlclose(lib._handle)
        _build.build(force=True)
        lib = ctypes.CDLL(LIB_PATH)
    for name, args in _SIGS.items():
        f = getattr(lib, name)
        f.argtypes = args
        f.restype = _RESTYPES.get(name, _i32)
    return lib


lib = _load()


def _wrap(name):
    f = getattr(lib, name)
    if name in _RESTYPES:
        return f

    def call(*args):
        st = f(*args)
        if st != MPS_OK:
            raise MpsError(st, name, (lib.mps_last_error() or b"").decode())
        return st
    call.__name__ = name
    call.__doc__ = "C-ABI %s (include/mpspmm.h); raises MpsError on a non-OK status." % name
    return call


for _n in _SIGS:
    globals()[_n] = _wrap(_n)

EXPORTED = tuple(_SIGS)
