"""ctypes declarations of include/mg.h (argument marshalling only)."""
from __future__ import annotations

import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# MG_LIB_VARIANT=<name> loads a diagnostics build libmg_<name>.so (build.py --variant <name>)
_VARIANT = os.environ.get("MG_LIB_VARIANT", "")
LIB_PATH = os.path.join(_HERE, f"libmg_{_VARIANT}.so" if _VARIANT else "libmg.so")

MG_OK, MG_ERR_INVALID_ARG, MG_ERR_UNSUPPORTED, MG_ERR_OUT_OF_MEMORY, MG_ERR_CUDA, MG_ERR_INTERNAL = range(6)
MG_BF16, MG_FP16 = 0, 1
STATUS_NAMES = {0: "OK", 1: "INVALID_ARG", 2: "UNSUPPORTED", 3: "OUT_OF_MEMORY", 4: "CUDA", 5: "INTERNAL"}

# Every symbol include/mg.h declares (checked by tests/test_abi.py).
EXPORTED = [
    "mg_plan_create", "mg_plan_create_ex", "mg_plan_create_batched", "mg_plan_destroy", "mg_last_error", "mg_plan_info_get",
    "mg_plan_export", "mg_sparse_attention_fwd", "mg_sparse_attention_fwd_host", "mg_selftest_umma",
    "mg_abi_version", "mg_plan_set_profiling", "mg_plan_get_profile", "mg_plan_get_profile_calls", "mg_plan_set_trace",
    "mg_sparse_attention_fwd_padded", "mg_staged_get_sizes", "mg_staged_sddmm", "mg_staged_softmax", "mg_staged_spmm", "mg_sparse_attention_fwd_staged", "mg_sparse_attention_fwd_staged_ex", "mg_plan_autotune",
]


class mg_tensor(C.Structure):
    _fields_ = [("data", C.c_void_p), ("dtype", C.c_int32), ("reserved", C.c_int32),
                ("batch", C.c_int64), ("heads", C.c_int64), ("seq_len", C.c_int64), ("head_dim", C.c_int64),
                ("stride_b", C.c_int64), ("stride_h", C.c_int64), ("stride_l", C.c_int64)]


class mg_plan_opts(C.Structure):
    _fields_ = [("block", C.c_int32), ("force_all_fine", C.c_int32), ("strip_max_cols", C.c_int32),
                ("num_sms", C.c_int32), ("fine_kernel", C.c_int32), ("concurrency", C.c_int32),
                ("tau", C.c_float), ("dense_chunk", C.c_int32)]


class mg_plan_info(C.Structure):
    _fields_ = [("L", C.c_int64), ("heads", C.c_int32), ("d", C.c_int32), ("window", C.c_int32),
                ("block", C.c_int32), ("n_row_blocks", C.c_int64), ("n_tiles", C.c_int64),
                ("n_full_tiles", C.c_int64), ("nnz_coarse", C.c_int64), ("nnz_fine", C.c_int64),
                ("n_global", C.c_int64), ("nnz_total", C.c_int64), ("n_fine_rows", C.c_int64),
                ("nnz_fine_strip", C.c_int64), ("nnz_fine_cuda", C.c_int64), ("n_items", C.c_int64),
                ("n_strip_tiles", C.c_int64), ("computed_scores", C.c_int64), ("kernels_per_fwd", C.c_int32),
                ("reserved", C.c_int32)]


class mg_profile(C.Structure):
    _fields_ = [("calls", C.c_int64), ("fine_ms", C.c_double), ("coarse_ms", C.c_double), ("total_ms", C.c_double)]


class mg_staged_sizes(C.Structure):
    _fields_ = [("tile_elems", C.c_int64), ("csr_elems", C.c_int64), ("global_elems", C.c_int64),
                ("ocsr_elems", C.c_int64), ("lpad", C.c_int64)]


_lib = None


def load() -> C.CDLL:
    """Load libmg.so. Raises (loudly) if the extension has not been built — there is no fallback."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} is missing: build it with `python -m paper_conf_iiswc_lica22_b200.build` "
                           "(there is no CPU fallback)")
    lib = C.CDLL(LIB_PATH)
    P = C.c_void_p
    i32p = C.POINTER(C.c_int32)
    lib.mg_plan_create.argtypes = [C.c_int64, C.c_int32, C.c_int32, C.c_int32, i32p, C.c_int64, i32p, C.c_int64,
                                   C.POINTER(P)]
    lib.mg_plan_create_ex.argtypes = [C.c_int64, C.c_int32, C.c_int32, C.c_int32, i32p, C.c_int64, i32p,
                                      C.c_int64, C.POINTER(mg_plan_opts), C.POINTER(P)]
    lib.mg_plan_create_batched.argtypes = [C.c_int64, C.c_int32, C.c_int32, C.c_int32, C.c_int64,
                                           C.POINTER(C.c_int64), i32p, C.POINTER(C.c_int64), i32p,
                                           C.POINTER(mg_plan_opts), C.POINTER(P)]
    lib.mg_plan_destroy.argtypes = [P]
    lib.mg_last_error.restype = C.c_char_p
    lib.mg_last_error.argtypes = []
    lib.mg_plan_info_get.argtypes = [P, C.POINTER(mg_plan_info)]
    lib.mg_plan_export.argtypes = [P, i32p, i32p, C.POINTER(C.c_uint64), i32p, i32p, i32p]
    tp = C.POINTER(mg_tensor)
    lib.mg_sparse_attention_fwd.argtypes = [P, tp, tp, tp, tp, P]
    lib.mg_sparse_attention_fwd_host.argtypes = [P, tp, tp, tp, tp, P]
    lib.mg_sparse_attention_fwd_padded.argtypes = [P, tp, tp, tp, tp, P, P]
    lib.mg_selftest_umma.argtypes = [C.c_int32, P, P, P, P]
    lib.mg_plan_set_profiling.argtypes = [P, C.c_int32]
    lib.mg_plan_get_profile.argtypes = [P, C.POINTER(mg_profile)]
    lib.mg_plan_get_profile_calls.argtypes = [P, C.POINTER(mg_profile), C.POINTER(C.c_double), C.c_int64]
    lib.mg_plan_set_trace.argtypes = [P, P, C.c_int64]
    lib.mg_staged_get_sizes.argtypes = [P, C.POINTER(mg_staged_sizes)]
    lib.mg_staged_sddmm.argtypes = [P, tp, tp, P, P, P, P]
    lib.mg_staged_softmax.argtypes = [P, C.c_int64, C.c_int32, P, P, P, P, P, P, P]
    lib.mg_staged_spmm.argtypes = [P, P, P, P, tp, tp, P, P]
    lib.mg_sparse_attention_fwd_staged.argtypes = [P, tp, tp, tp, tp, P]
    lib.mg_sparse_attention_fwd_staged_ex.argtypes = [P, tp, tp, tp, tp, C.c_int32, P]
    lib.mg_plan_autotune.argtypes = [C.c_int64, C.c_int32, C.c_int32, C.c_int32, i32p, C.c_int64, i32p, C.c_int64,
                                     tp, tp, tp, tp, P, C.POINTER(P), C.POINTER(mg_plan_opts), C.POINTER(C.c_double)]
    lib.mg_abi_version.restype = C.c_int32
    lib.mg_abi_version.argtypes = []
    for name in EXPORTED:
        if name != "mg_last_error" and name != "mg_abi_version":
            getattr(lib, name).restype = C.c_int
    _lib = lib
    return lib


class MGError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"mg status {STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


def check(status: int) -> None:
    if status != MG_OK:
        raise MGError(status, load().mg_last_error().decode())
