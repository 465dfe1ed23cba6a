"""ctypes binding of libatos.so (include/atos.h).  Argument marshalling only.

No CPU fallback exists: if the shared library cannot be loaded, or a call
returns an error, a RuntimeError is raised.
"""
from __future__ import annotations

import ctypes
import os
import threading

HERE = os.path.dirname(os.path.abspath(__file__))
# ATOS_LIB selects an experimental variant build (tools only); the default is the in-tree library
LIB_PATH = os.environ.get("ATOS_LIB") or os.path.join(HERE, "libatos.so")

ATOS_OK = 0
ERRORS = {
    -1: "ATOS_ERR_INVALID_ARG", -2: "ATOS_ERR_OOM", -3: "ATOS_ERR_CUDA", -4: "ATOS_ERR_NCCL",
    -5: "ATOS_ERR_QUEUE_OVERFLOW", -6: "ATOS_ERR_TIMEOUT", -7: "ATOS_ERR_NOT_SYMMETRIC",
    -8: "ATOS_ERR_UNSUPPORTED",
}
MEM_HOST, MEM_DEVICE = 0, 1
UNREACHED = 0xFFFFFFFF
COMM_ID_BYTES = 128

# every symbol include/atos.h declares (checked by tests/test_abi.py)
EXPORTS = [
    "atos_cfg_default", "atos_csr_create", "atos_csr_destroy", "atos_csr_info", "atos_bfs",
    "atos_pagerank", "atos_color", "atos_comm_unique_id", "atos_comm_create", "atos_comm_destroy",
    "atos_csr_create_part", "atos_partition_range", "atos_last_error", "atos_version",
    "atos_kernel_launches", "atos_bfs_bsp", "atos_pagerank_bsp", "atos_color_bsp", "atos_csr_create_ex", "atos_csr_layout", "atos_comm_create_host", "atos_comm_gather",
]
LAYOUT_AUTO, LAYOUT_INPUT, LAYOUT_DEGREE = 0, 1, 2

# atos_host_alltoallv_fn / atos_host_allreduce_fn (include/atos.h)
HOST_A2A_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.POINTER(ctypes.c_uint64),
                               ctypes.c_void_p, ctypes.POINTER(ctypes.c_uint64))
HOST_AR_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int)


class Stats(ctypes.Structure):
    _fields_ = [
        ("pops", ctypes.c_uint64), ("pushes", ctypes.c_uint64), ("edges", ctypes.c_uint64),
        ("rounds", ctypes.c_uint64), ("bytes_exchanged", ctypes.c_uint64), ("kernel_ms", ctypes.c_double),
        ("residual_sum", ctypes.c_double), ("colors_used", ctypes.c_int64), ("worker_ms", ctypes.c_double),
        ("timeline_len", ctypes.c_uint64), ("flags", ctypes.c_uint64), ("max_queue_occupancy", ctypes.c_uint64),
    ]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_ }


class Cfg(ctypes.Structure):
    _fields_ = [
        ("struct_size", ctypes.c_uint32), ("persistent", ctypes.c_int), ("worker", ctypes.c_int),
        ("fetch_size", ctypes.c_int), ("num_blocks", ctypes.c_int), ("block_threads", ctypes.c_int),
        ("dedupe", ctypes.c_int), ("check_size", ctypes.c_int), ("conflict_policy", ctypes.c_int),
        ("permute_init", ctypes.c_int), ("validate", ctypes.c_int), ("out_where", ctypes.c_int),
        ("queue_capacity", ctypes.c_uint64), ("timeout_s", ctypes.c_double), ("stream", ctypes.c_void_p),
        ("stats", ctypes.POINTER(Stats)), ("l2_persist", ctypes.c_int), ("big_threshold", ctypes.c_int),
        ("big_chunk", ctypes.c_int), ("timeline_cap", ctypes.c_uint32), ("timeline", ctypes.c_void_p),
        ("timeline_interval_ns", ctypes.c_uint32), ("depth_state", ctypes.c_int), ("engine_variant", ctypes.c_int),
        ("barrier_free", ctypes.c_int), ("recolor_spread", ctypes.c_int),
    ]


_lock = threading.Lock()
_lib = None


def load(build_if_missing: bool = True):
    """Load libatos.so (building it first with nvcc when missing/stale and nvcc exists)."""
    global _lib
    with _lock:
        if _lib is not None:
            return _lib
        if build_if_missing and not os.environ.get("ATOS_LIB") and os.path.exists("/usr/local/cuda/bin/nvcc"):
            from . import build_lib
            build_lib.build()
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"libatos.so not found at {LIB_PATH}; run __graft_entry__.build()")
        lib = ctypes.CDLL(LIB_PATH, mode=ctypes.RTLD_GLOBAL)
        P, i64, i32, u64, dbl, sz = (ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_uint64,
                                     ctypes.c_double, ctypes.c_size_t)
        sig = {
            "atos_cfg_default": (None, [ctypes.POINTER(Cfg)]),
            "atos_csr_create": (i32, [ctypes.POINTER(P), i64, i64, P, P, i32, i32, i32]),
            "atos_csr_create_ex": (i32, [ctypes.POINTER(P), i64, i64, P, P, i32, i32, i32, i32]),
            "atos_csr_destroy": (None, [P]),
            "atos_csr_info": (i32, [P, ctypes.POINTER(i64), ctypes.POINTER(i64), ctypes.POINTER(i32)]),
            "atos_csr_layout": (i32, [P, ctypes.POINTER(i32)]),
            "atos_bfs": (i32, [P, i64, P, ctypes.POINTER(Cfg)]),
            "atos_pagerank": (i32, [P, dbl, dbl, P, ctypes.POINTER(Cfg)]),
            "atos_color": (i32, [P, u64, P, ctypes.POINTER(Cfg)]),
            "atos_bfs_bsp": (i32, [P, i64, P, ctypes.POINTER(Cfg)]),
            "atos_pagerank_bsp": (i32, [P, dbl, dbl, P, ctypes.POINTER(Cfg)]),
            "atos_color_bsp": (i32, [P, u64, P, ctypes.POINTER(Cfg)]),
            "atos_comm_unique_id": (i32, [P, sz]),
            "atos_comm_create": (i32, [ctypes.POINTER(P), i32, i32, P, sz, i32]),
            "atos_comm_destroy": (None, [P]),
            "atos_comm_gather": (i32, [P, i64, P, sz, P, P]),
            "atos_comm_create_host": (i32, [ctypes.POINTER(P), i32, i32, i32, HOST_A2A_FN, HOST_AR_FN, P]),
            "atos_csr_create_part": (i32, [ctypes.POINTER(P), P, i64, i64, i64, i64, P, P, i32]),
            "atos_partition_range": (i32, [i64, i32, i32, ctypes.POINTER(i64), ctypes.POINTER(i64)]),
            "atos_last_error": (ctypes.c_char_p, []),
            "atos_version": (i32, []),
            "atos_kernel_launches": (u64, []),
        }
        for name, (res, args) in sig.items():
            f = getattr(lib, name)
            f.restype = res
            f.argtypes = args
        _lib = lib
        return lib


def check(rc: int, what: str):
    if rc != ATOS_OK:
        msg = load().atos_last_error().decode(errors="replace")
        raise RuntimeError(f"{what} failed: {ERRORS.get(rc, rc)}: {msg}")


def default_cfg(**knobs) -> Cfg:
    cfg = Cfg()
    load().atos_cfg_default(ctypes.byref(cfg))
    for k, v in knobs.items():
        if not hasattr(cfg, k):
            raise TypeError(f"unknown atos_cfg field {k!r}")
        setattr(cfg, k, v)
    return cfg
