"""ctypes binding of libms.so (include/ms.h): argument marshalling only.

Every step of the multisplit runs in the CUDA kernels behind this ABI; there
is no fallback.  If the library is missing the import of any entry point
raises, loudly.
"""
from __future__ import annotations

import ctypes
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libms.so")

MS_OK = 0
MS_ERR_INVALID_ARG = -1
MS_ERR_UNSUPPORTED = -2
MS_ERR_ALIGNMENT = -3
MS_ERR_ALIAS = -4
MS_ERR_WORKSPACE = -5
MS_ERR_CUDA = -6
MS_ERR_NCCL = -7
MS_ERR_BUCKET_RANGE = -8

MS_LOWBITS, MS_DELTA, MS_SPLITTERS, MS_IDS = 0, 1, 2, 3
MS_VALIDATE, MS_VARIANT_3K, MS_VARIANT_RANGED, MS_VARIANT_ONE, MS_ABLATION_DIRECT = 1, 2, 4, 8, 16
MS_ABLATION_NW2, MS_ABLATION_NW4, MS_ABLATION_BALLOT, MS_ABLATION_WARP = 32, 64, 128, 256
# ms_plan_geometry's variant codes and the kernel launches one ms_run of each enqueues
VARIANT_TILE, VARIANT_RANGED, VARIANT_ONE, VARIANT_WIDE = 0, 1, 2, 3   # WIDE: m > 256, two passes
LAUNCHES = {VARIANT_TILE: 3, VARIANT_RANGED: 2, VARIANT_ONE: 1}

# every symbol include/ms.h declares (tests check the library exports them all)
EXPORTS = [
    "ms_plan_create", "ms_plan_workspace_size", "ms_plan_geometry", "ms_run",
    "ms_plan_workspace_size_host", "ms_run_host", "ms_prescan", "ms_scan", "ms_postscan",
    "ms_bucket_ids", "ms_plan_check", "ms_plan_destroy", "ms_status_string",
    "ms_plan_last_launches", "ms_plan_trace", "ms_plan_trace_read", "ms_dist_pieces",
    "ms_dist_targets", "ms_postscan_scatter", "ms_plan_spec", "ms_dist_workspace_size", "ms_dist_run",
    "ms_nccl_get_unique_id", "ms_nccl_comm_init", "ms_nccl_comm_destroy", "ms_dist_workspace_size_fused",
    "ms_dist_run_fused",
]

MS_MAX_PEERS = 8


class ms_scatter_target(ctypes.Structure):
    _fields_ = [
        ("nranks", ctypes.c_int32),
        ("pad_", ctypes.c_int32),
        ("keys_dst", ctypes.c_void_p * MS_MAX_PEERS),
        ("vals_dst", ctypes.c_void_p * MS_MAX_PEERS),
        ("win_start", ctypes.c_uint64 * (MS_MAX_PEERS + 1)),
        ("delta", ctypes.c_uint64 * 32),
    ]


class ms_bucket_spec(ctypes.Structure):
    _fields_ = [
        ("kind", ctypes.c_int32),
        ("m", ctypes.c_uint32),
        ("shift", ctypes.c_uint32),
        ("delta", ctypes.c_uint32),
        ("splitters", ctypes.POINTER(ctypes.c_uint32)),
        ("id_bytes", ctypes.c_uint32),
    ]


class MultisplitError(RuntimeError):
    def __init__(self, status: int, what: str = ""):
        self.status = status
        super().__init__(f"{what}: {status_string(status)} ({status})")


_lib = None


def lib():
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"libms.so not built ({LIB_PATH}); run __graft_entry__.build() -- "
                          "there is no CPU fallback for the multisplit")
    L = ctypes.CDLL(LIB_PATH)
    P, U32, U64, I32, SZ = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int32, ctypes.c_size_t
    L.ms_plan_create.argtypes = [ctypes.POINTER(P), ctypes.POINTER(ms_bucket_spec), U64, ctypes.c_int, U32,
                                 ctypes.c_int]
    L.ms_plan_workspace_size.argtypes = [P, U64, ctypes.POINTER(SZ)]
    L.ms_plan_workspace_size_host.argtypes = [P, U64, ctypes.POINTER(SZ)]
    L.ms_plan_geometry.argtypes = [P, U64, ctypes.POINTER(U32), ctypes.POINTER(U64), ctypes.POINTER(I32)]
    L.ms_run.argtypes = [P, P, P, P, P, P, U64, P, P, SZ, P]
    L.ms_run_host.argtypes = [P, P, P, P, P, P, U64, P, P, SZ, P]
    L.ms_prescan.argtypes = [P, P, P, U64, P, P, SZ, P]
    L.ms_scan.argtypes = [P, P, U64, P, P, SZ, P]
    L.ms_postscan.argtypes = [P, P, P, P, P, P, P, U64, P, SZ, P]
    L.ms_bucket_ids.argtypes = [P, P, U64, P, P]
    L.ms_plan_check.argtypes = [P, P, P]
    L.ms_plan_destroy.argtypes = [P]
    L.ms_status_string.argtypes = [I32]
    L.ms_status_string.restype = ctypes.c_char_p
    L.ms_plan_last_launches.argtypes = [P]
    L.ms_plan_trace.argtypes = [P, ctypes.c_int]
    L.ms_plan_trace_read.argtypes = [P, P, I32, ctypes.POINTER(I32), ctypes.POINTER(I32)]
    L.ms_dist_pieces.argtypes = [I32, I32, U32, P, P, I32, ctypes.POINTER(I32), P, I32, ctypes.POINTER(I32), P,
                                 ctypes.POINTER(U64), ctypes.POINTER(U64)]
    L.ms_dist_targets.argtypes = [I32, I32, U32, P, P, P]
    L.ms_postscan_scatter.argtypes = [P, P, P, P, U64, ctypes.POINTER(ms_scatter_target), P, SZ, P]
    L.ms_plan_spec.argtypes = [P, ctypes.POINTER(ms_bucket_spec), ctypes.POINTER(I32)]
    L.ms_dist_workspace_size.argtypes = [P, U64, I32, ctypes.POINTER(SZ)]
    L.ms_dist_run.argtypes = [P, P, P, P, P, U64, P, P, U64, P, ctypes.POINTER(U64), ctypes.POINTER(U64), P, SZ, P]
    L.ms_dist_workspace_size_fused.argtypes = [P, U64, I32, ctypes.POINTER(SZ)]
    L.ms_dist_run_fused.argtypes = [P, P, P, P, U64, P, P, U64, P, ctypes.POINTER(U64), ctypes.POINTER(U64), P,
                                    SZ, P]
    L.ms_nccl_get_unique_id.argtypes = [P]
    L.ms_nccl_comm_init.argtypes = [ctypes.POINTER(P), I32, I32, P, ctypes.c_int]
    L.ms_nccl_comm_destroy.argtypes = [P]
    for name in EXPORTS:
        f = getattr(L, name)
        if name != "ms_status_string":
            f.restype = I32
    _lib = L
    return L


def status_string(s: int) -> str:
    try:
        return lib().ms_status_string(int(s)).decode()
    except ImportError:
        return "libms.so missing"


def check(status: int, what: str):
    if status != MS_OK:
        raise MultisplitError(status, what)
