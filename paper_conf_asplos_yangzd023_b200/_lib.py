"""ctypes declarations of include/betty.h (libbetty.so).  Marshalling only.

The shared library is REQUIRED: importing a function from here on a machine
without libbetty.so raises; there is no CPU or PyTorch fallback.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# BETTY_LIB_PATH: an alternative build of the same library (tuning sweeps only, tools/sweep_g4.sh)
LIB_PATH = os.environ.get("BETTY_LIB_PATH") or os.path.join(_HERE, "libbetty.so")

i32, i64, f32, vp = ctypes.c_int32, ctypes.c_int64, ctypes.c_float, ctypes.c_void_p
P_i32 = ctypes.POINTER(ctypes.c_int32)


class betty_block(ctypes.Structure):
    _fields_ = [("n_dst", i64), ("n_src", i64), ("n_edges", i64), ("indptr", vp), ("indices", vp),
                ("src_pos", vp), ("src_gid", vp), ("t_indptr", vp), ("t_indices", vp)]


class betty_csr(ctypes.Structure):
    _fields_ = [("n", i64), ("nnz", i64), ("indptr", vp), ("col", vp), ("w", vp)]


class betty_model(ctypes.Structure):
    _fields_ = [("L", i32), ("aggr", i32), ("gemm", i32), ("feat_dtype", i32), ("dims", P_i32)]


class betty_plan_info(ctypes.Structure):
    _fields_ = [("n_groups", i32), ("L", i32), ("edges", i64 * 16), ("n_src", i64 * 16), ("n_dst", i64 * 16),
                ("max_group_edges", i64 * 16), ("reg_nnz", i64), ("arena_bytes", i64),
                ("kernels_per_step", i32)]


STATUS = {0: "BETTY_OK", 1: "BETTY_EINVAL", 2: "BETTY_ENOMEM", 3: "BETTY_ECUDA", 4: "BETTY_EOVERFLOW",
          5: "BETTY_EUNSUPPORTED"}

_lib = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"libbetty.so not built ({LIB_PATH}); run `make -C paper_conf_asplos_yangzd023_b200` "
                           "or __graft_entry__.build() -- there is no fallback path")
    L = ctypes.CDLL(LIB_PATH)
    pp = ctypes.POINTER
    sigs = {
        "betty_version": (ctypes.c_char_p, []),
        "betty_ctx_create": (i32, [ctypes.c_int, vp, vp, vp, pp(vp)]),
        "betty_ctx_destroy": (None, [vp]),
        "betty_last_error": (ctypes.c_char_p, [vp]),
        "betty_num_params": (i64, [pp(betty_model)]),
        "betty_reg_build": (i32, [vp, pp(betty_block), pp(betty_csr), vp]),
        "betty_reg_build_rows": (i32, [vp, pp(betty_block), i64, i64, pp(betty_csr), vp]),
        "betty_csr_free": (None, [vp, pp(betty_csr)]),
        "betty_extract_blocks": (i32, [vp, pp(betty_block), i32, vp, i64, i32, i32, pp(betty_block), vp]),
        "betty_block_free": (None, [vp, pp(betty_block), i32]),
        "betty_sage_fwd": (i32, [vp, pp(betty_model), vp, pp(betty_block), vp, i64, pp(vp), vp, vp]),
        "betty_sage_bwd": (i32, [vp, pp(betty_model), vp, pp(betty_block), vp, vp, f32, vp, vp, vp]),
        "betty_saved_free": (None, [vp, vp]),
        "betty_plan_create": (i32, [vp, pp(betty_model), pp(betty_block), i32, vp, i64, i32, P_i32, i32, i32, i32,
                                    pp(vp), vp]),
        "betty_plan_info_get": (i32, [vp, pp(betty_plan_info)]),
        "betty_plan_destroy": (None, [vp, vp]),
        "betty_plan_set_reg_rows": (i32, [vp, vp, i64, i64, vp]),
        "betty_plan_set_feature_shards": (i32, [vp, vp, i32, vp, i64]),
        "betty_dev_alloc": (i32, [vp, ctypes.c_size_t, pp(vp)]),
        "betty_dev_free": (i32, [vp, vp]),
        "betty_ipc_handle": (i32, [vp, vp, vp]),
        "betty_ipc_open": (i32, [vp, vp, pp(vp)]),
        "betty_ipc_close": (i32, [vp, vp]),
        "betty_step": (i32, [vp, vp, vp, vp, i64, vp, f32, vp, vp, vp]),
        "betty_adam": (i32, [vp, vp, vp, vp, vp, i64, i32, f32, f32, f32, f32, i32, vp]),
        "betty_sync_check": (i32, [vp, vp]),
        "betty_reg_partition": (i32, [vp, vp, vp, i64, i32, vp]),
        "betty_plan_probe": (i32, [vp, i32]),
        "betty_plan_group_blocks": (i32, [vp, vp, i32, pp(betty_block), vp]),
        "betty_test_gemm": (i32, [vp, i32, vp, i64, vp, i64, i64, i64, i32, i32, vp, i64, i32, vp]),
        "betty_plan_probe_read": (i32, [vp, pp(f32), pp(i32)]),
        "betty_reg_partition_ex": (i32, [vp, vp, vp, i64, i32, i32, ctypes.c_double, vp]),
        "betty_mb_sizes": (i32, [vp, pp(betty_block), i32, vp, i64, i32, vp, vp]),
        "betty_mem_estimate": (i32, [pp(betty_model), vp, vp]),
        "betty_memory_aware_k": (i32, [vp, pp(betty_model), pp(betty_block), i32, vp, vp, vp, i64, i64, i32, i32,
                                       i32, vp, pp(i32), pp(i64), vp]),
    }
    for name, (res, args) in sigs.items():
        fn = getattr(L, name)
        fn.restype = res
        fn.argtypes = args
    _lib = L
    return L


EXPORTED = ["betty_version", "betty_ctx_create", "betty_ctx_destroy", "betty_last_error", "betty_num_params",
            "betty_reg_build", "betty_csr_free", "betty_extract_blocks", "betty_block_free", "betty_sage_fwd",
            "betty_sage_bwd", "betty_saved_free", "betty_plan_create", "betty_plan_info_get", "betty_plan_destroy",
            "betty_step", "betty_adam", "betty_sync_check", "betty_reg_partition", "betty_plan_probe",
            "betty_plan_probe_read", "betty_plan_group_blocks", "betty_test_gemm", "betty_mb_sizes",
            "betty_mem_estimate", "betty_memory_aware_k", "betty_reg_partition_ex", "betty_reg_build_rows",
            "betty_plan_set_reg_rows", "betty_plan_set_feature_shards", "betty_dev_alloc", "betty_dev_free",
            "betty_ipc_handle", "betty_ipc_open", "betty_ipc_close"]
