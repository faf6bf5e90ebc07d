"""ctypes binding of libwg.so (include/wg.h).  Argument marshalling only; every
step of the path runs in the library's sm_100a kernels.  There is no fallback:
if the library is missing this module raises."""

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libwg.so")

WG_OK = 0
STATUS = {0: "WG_OK", 1: "WG_ERR_INVALID_ARG", 2: "WG_ERR_CUDA", 3: "WG_ERR_OOM", 4: "WG_ERR_PEER_ACCESS",
          5: "WG_ERR_CAPACITY", 6: "WG_ERR_UNSUPPORTED", 7: "WG_ERR_COLLECTIVE"}
DEVERR = {0x1: "ID_RANGE", 0x2: "DUP_TARGET", 0x4: "CAPACITY", 0x8: "DEGREE", 0x10: "EPOCH"}
WG_MAX_WORLD = 8

ALLGATHER_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p)


class WgDsmDesc(ctypes.Structure):
    _fields_ = [("rank", ctypes.c_int32), ("world_size", ctypes.c_int32), ("device", ctypes.c_int32),
                ("feat_dtype", ctypes.c_int32), ("num_nodes", ctypes.c_int64), ("local_num_edges", ctypes.c_int64),
                ("feat_dim", ctypes.c_int64), ("max_batch_keys", ctypes.c_int64), ("allgather", ALLGATHER_FN),
                ("ctx", ctypes.c_void_p), ("flags", ctypes.c_uint32), ("reserved", ctypes.c_uint32)]


# wg_dsm_desc.flags (include/wg.h)
WG_DSM_WHOLE_ROWS = 0x1
WG_DSM_WIDE_HASH = 0x2
WG_DSM_PAD64 = 0x4
WG_DSM_CSR_REPLICATED = 0x8
WG_DSM_COL32 = 0x10
WG_DSM_HASHED = 0x20

# wg_dsm_unique_format (include/wg.h)
WG_UNIQUE_WIDE, WG_UNIQUE_COMPACT, WG_UNIQUE_DIRECT = 0, 1, 2


class WgError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


_lib = None


def lib():
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'` "
                          "(there is no CPU fallback)")
    L = ctypes.CDLL(LIB_PATH)
    P, I32, I64, U64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64
    L.wg_dsm_create.argtypes = [ctypes.POINTER(WgDsmDesc), ctypes.POINTER(P)]
    L.wg_dsm_local_view.argtypes = [P, P, P, P, P, P]
    L.wg_dsm_shard_info.argtypes = [P, I32, P, P]
    L.wg_dsm_feat_layout.argtypes = [P, P, P, P, P]
    L.wg_dsm_destroy.argtypes = [P]
    L.wg_dsm_fork.argtypes = [P, I64, P]
    L.wg_sample_neighbors.argtypes = [P, P, I64, P, I32, U64, P, I32, P, P, P, P, P]
    L.wg_append_unique.argtypes = [P, P, I64, P, P, I64, P, P, P, P, P, P]
    L.wg_sample_hop.argtypes = [P, P, I64, P, I32, U64, P, I32, P, P, P, P, P, P, P, P, P, P]
    L.wg_gather.argtypes = [P, P, I64, P, P, P]
    L.wg_gather_rows.argtypes = [P, P, I64, P, P, P, I64, P]
    L.wg_dsm_chase.argtypes = [P, I32, I64, I64, P, P]
    L.wg_bucket_by_owner.argtypes = [P, P, I64, P, P, P, P, P]
    L.wg_rows_permute.argtypes = [P, P, P, I64, I64, P]
    L.wg_spmm_mean_forward.argtypes = [P, I64, P, P, P, I64, I64, P, P]
    L.wg_spmm_mean_backward.argtypes = [P, I64, P, P, P, P, I64, P, I64, P]
    L.wg_device_error.argtypes = [P, P, I32]
    L.wg_dsm_reset_workspace.argtypes = [P, P]
    L.wg_dsm_set_gather_occupancy.argtypes = [P, I32]
    L.wg_dsm_debug_set_epoch.argtypes = [P, ctypes.c_uint32]
    L.wg_dsm_set_stage_events.argtypes = [P, P, I32]
    L.wg_dsm_unique_format.argtypes = [P, P, P]
    L.wg_micro_random_read.argtypes = [P, I64, I32, I32, I32, P, P, P]
    L.wg_micro_atomics.argtypes = [P, I64, I32, I32, I32, P, P, P]
    for f in ("wg_dsm_create", "wg_dsm_fork", "wg_dsm_local_view", "wg_dsm_shard_info", "wg_dsm_feat_layout",
              "wg_dsm_destroy", "wg_sample_neighbors", "wg_append_unique", "wg_sample_hop", "wg_gather", "wg_gather_rows",
              "wg_dsm_chase", "wg_spmm_mean_forward", "wg_spmm_mean_backward", "wg_bucket_by_owner", "wg_rows_permute",
              "wg_device_error", "wg_dsm_reset_workspace", "wg_dsm_set_gather_occupancy",
              "wg_dsm_debug_set_epoch", "wg_micro_random_read", "wg_micro_atomics", "wg_dsm_set_stage_events",
              "wg_dsm_unique_format"):
        getattr(L, f).restype = ctypes.c_int
    L.wg_last_error.restype = ctypes.c_char_p
    L.wg_last_error.argtypes = []
    L.wg_version.restype = ctypes.c_char_p
    L.wg_version.argtypes = []
    _lib = L
    return L


def check(status):
    if status != WG_OK:
        raise WgError(status, lib().wg_last_error().decode())


EXPORTS = ["wg_dsm_create", "wg_dsm_fork", "wg_dsm_local_view", "wg_dsm_shard_info", "wg_dsm_feat_layout", "wg_dsm_destroy", "wg_sample_neighbors",
           "wg_append_unique", "wg_sample_hop", "wg_gather", "wg_gather_rows", "wg_dsm_chase", "wg_spmm_mean_forward",
           "wg_spmm_mean_backward", "wg_bucket_by_owner", "wg_rows_permute", "wg_device_error", "wg_dsm_reset_workspace", "wg_dsm_set_gather_occupancy",
           "wg_dsm_debug_set_epoch", "wg_micro_random_read", "wg_micro_atomics", "wg_dsm_set_stage_events", "wg_dsm_unique_format", "wg_last_error", "wg_version"]
