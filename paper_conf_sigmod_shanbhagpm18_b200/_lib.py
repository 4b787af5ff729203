"""ctypes binding of include/topk.h (argument marshalling only).

Every step of the top-k runs in libtopk_b200.so's sm_100a kernels; torch provides the
device memory and the current CUDA stream.  There is no CPU fallback: if the library
cannot be loaded the call raises.
"""
from __future__ import annotations

import ctypes
import os

from . import _build

TOPK_OK = 0
STATUS = {0: "TOPK_OK", 1: "TOPK_ERR_INVALID_ARG", 2: "TOPK_ERR_UNSUPPORTED",
          3: "TOPK_ERR_WORKSPACE", 4: "TOPK_ERR_CUDA", 5: "TOPK_ERR_NCCL"}
F32, U32, F64 = 0, 1, 2
LARGEST, SMALLEST = 0, 1
MODE_FILTER, MODE_PURE = 0, 1

# Every symbol include/topk.h declares (tests check the .so exports all of them).
SYMBOLS = (
    "topk_workspace_bytes", "topk_workspace_init", "topk_select", "topk_f32", "topk_u32",
    "topk_f64", "topk_u32_kv", "topk_f64_kv", "topk_merge_workspace_bytes", "topk_merge", "topk_merge_sorted",
    "topk_launch_count", "topk_status_string", "topk_abi_version", "topk_probe_read",
    "topk_host_workspace_bytes", "topk_select_host", "topk_nccl_unique_id", "topk_nccl_comm_init",
    "topk_nccl_comm_destroy", "topk_sharded_workspace_bytes", "topk_select_sharded",
    "topk_f32_sharded", "topk_query", "topk_kk", "topk_kkk", "topk_radix_workspace_bytes", "topk_radix",
)
PRED_RANGE, PRED_IN = 1, 2


class Pred(ctypes.Structure):
    """topk_pred_t (include/topk.h)."""
    _fields_ = [("kind", ctypes.c_int), ("col", ctypes.c_void_p), ("lo", ctypes.c_uint32),
                ("hi", ctypes.c_uint32), ("in_mask", ctypes.c_uint64)]

_lib = None


class TopkError(RuntimeError):
    pass


def load(build_if_missing: bool = True):
    """Load libtopk_b200.so (building it in-tree first if missing or stale)."""
    global _lib
    if _lib is not None:
        return _lib
    path = os.environ.get("TOPK_LIB")  # dev: load an alternative in-tree build
    if path is None:
        if build_if_missing:
            _build.build()
        path = _build.LIB
    if not os.path.exists(path):
        raise TopkError(f"CUDA library missing: {path} (run __graft_entry__.build())")
    lib = ctypes.CDLL(path)
    vp, u64, u32, i32, sz = (ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int,
                             ctypes.c_size_t)
    lib.topk_workspace_bytes.argtypes = [i32, u64, u32]
    lib.topk_workspace_bytes.restype = sz
    lib.topk_workspace_init.argtypes = [vp, sz, vp]
    lib.topk_workspace_init.restype = i32
    lib.topk_select.argtypes = [i32, vp, vp, u64, u64, u32, i32, i32, vp, vp, vp, vp, sz, vp]
    lib.topk_select.restype = i32
    for name in ("topk_f32", "topk_u32", "topk_f64"):
        getattr(lib, name).argtypes = [vp, u64, u32, i32, vp, vp, vp, sz, vp]
        getattr(lib, name).restype = i32
    for name in ("topk_u32_kv", "topk_f64_kv"):
        getattr(lib, name).argtypes = [vp, vp, u64, u32, i32, vp, vp, vp, vp, sz, vp]
        getattr(lib, name).restype = i32
    lib.topk_merge_workspace_bytes.argtypes = [i32, u32, u32, u32]
    lib.topk_merge_workspace_bytes.restype = sz
    lib.topk_merge.argtypes = [i32, vp, vp, vp, u32, u32, u32, i32, vp, vp, vp, vp, sz, vp]
    lib.topk_merge.restype = i32
    lib.topk_merge_sorted.argtypes = [i32, vp, vp, vp, u32, u32, u32, i32, vp, vp, vp, vp, sz, vp]
    lib.topk_merge_sorted.restype = i32
    lib.topk_probe_read.argtypes = [vp, sz, i32, i32, i32, i32, vp, vp]
    lib.topk_probe_read.restype = i32
    lib.topk_host_workspace_bytes.argtypes = [i32, u64, u32, u64]
    lib.topk_host_workspace_bytes.restype = sz
    lib.topk_select_host.argtypes = [i32, vp, u64, u32, i32, vp, vp, u64, vp, sz, vp]
    lib.topk_select_host.restype = i32
    lib.topk_nccl_unique_id.argtypes = [vp]
    lib.topk_nccl_unique_id.restype = i32
    lib.topk_nccl_comm_init.argtypes = [vp, i32, i32, ctypes.POINTER(ctypes.c_void_p)]
    lib.topk_nccl_comm_init.restype = i32
    lib.topk_nccl_comm_destroy.argtypes = [vp]
    lib.topk_nccl_comm_destroy.restype = i32
    lib.topk_sharded_workspace_bytes.argtypes = [i32, u64, u32, i32]
    lib.topk_sharded_workspace_bytes.restype = sz
    lib.topk_select_sharded.argtypes = [i32, vp, vp, u64, u64, u32, i32, vp, vp, vp, vp, vp, sz,
                                        vp]
    lib.topk_select_sharded.restype = i32
    lib.topk_f32_sharded.argtypes = [vp, u64, u64, u32, i32, vp, vp, vp, vp, sz, vp]
    lib.topk_f32_sharded.restype = i32
    lib.topk_query.argtypes = [i32, vp, vp, ctypes.c_float, ctypes.POINTER(Pred), vp, u64, u32,
                               i32, vp, vp, vp, vp, sz, vp]
    lib.topk_query.restype = i32
    lib.topk_kk.argtypes = [vp, vp, ctypes.POINTER(Pred), vp, u64, u32, i32, i32, vp, vp, vp, vp,
                            vp, sz, vp]
    lib.topk_kk.restype = i32
    lib.topk_kkk.argtypes = [vp, vp, vp, ctypes.POINTER(Pred), vp, u64, u32, i32, i32, i32, vp, vp,
                             vp, vp, vp, vp, sz, vp]
    lib.topk_kkk.restype = i32
    lib.topk_radix_workspace_bytes.argtypes = [i32, u64, u32]
    lib.topk_radix_workspace_bytes.restype = sz
    lib.topk_radix.argtypes = [i32, vp, u64, u32, i32, vp, vp, vp, sz, vp]
    lib.topk_radix.restype = i32
    lib.topk_launch_count.argtypes = []
    lib.topk_launch_count.restype = u64
    lib.topk_status_string.argtypes = [i32]
    lib.topk_status_string.restype = ctypes.c_char_p
    lib.topk_abi_version.argtypes = []
    lib.topk_abi_version.restype = i32
    _lib = lib
    return lib


def check(status: int, what: str):
    if status != TOPK_OK:
        msg = load().topk_status_string(status).decode()
        raise TopkError(f"{what}: {msg}")
