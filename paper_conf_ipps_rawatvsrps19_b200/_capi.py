"""ctypes declarations of include/sdag.h (argument marshalling only).

Loads the in-tree ``lib/libsdag.so``.  There is no fallback: if the library
is missing the import of the product API fails loudly.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "lib", "libsdag.so")

c_i32, c_i64, c_dbl, c_char_p, c_void_p = ctypes.c_int32, ctypes.c_int64, ctypes.c_double, ctypes.c_char_p, ctypes.c_void_p
c_i64p = ctypes.POINTER(c_i64)
c_dblp = ctypes.POINTER(c_dbl)


class PlanOpts(ctypes.Structure):
    _fields_ = [("order", c_i32), ("device", c_i32), ("tune", c_i32), ("batch", c_i32),
                ("force_variant", c_char_p), ("fusion", c_i32), ("time_tile", c_i32)]


class PlanInfo(ctypes.Structure):
    _fields_ = [("n_arrays3d", c_i32), ("n_arrays1d", c_i32), ("n_scalars", c_i32),
                ("n_in", c_i32), ("n_out", c_i32), ("n_inout", c_i32),
                ("n_statements", c_i32), ("n_temporaries", c_i32),
                ("radius", c_i32 * 3), ("dims", c_i64 * 3), ("lo", c_i64 * 3), ("hi", c_i64 * 3),
                ("points", c_i64), ("flops_per_point", c_dbl), ("bytes_per_point", c_dbl), ("oi_paper", c_dbl),
                ("n_kernels", c_i32), ("n_variants", c_i32), ("dag", c_char_p), ("variant", c_char_p)]


SDAG_DEVICE_CURRENT = -1
SDAG_DEVICE_NONE = -2

STATUS = {0: "OK", 1: "INVALID_ARG", 2: "PARSE", 3: "SEMANTIC", 4: "UNSUPPORTED", 5: "DOMAIN", 6: "DEVICE",
          7: "CUDA", 8: "NCCL", 9: "NOMEM"}

_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"libsdag.so not built ({LIB_PATH}); run `make` or __graft_entry__.build()")
        L = ctypes.CDLL(LIB_PATH, mode=ctypes.RTLD_GLOBAL)
        S = c_i32  # sdag_status
        P = c_void_p  # handles
        sig = {
            "sdag_plan_opts_init": (None, [ctypes.POINTER(PlanOpts)]),
            "sdag_plan_create": (S, [c_char_p, c_i64p, ctypes.POINTER(PlanOpts), ctypes.POINTER(P)]),
            "sdag_plan_info_get": (S, [P, ctypes.POINTER(PlanInfo)]),
            "sdag_plan_arg": (S, [P, c_i32, c_i32, ctypes.POINTER(c_char_p), ctypes.POINTER(c_i32)]),
            "sdag_plan_variant_name": (S, [P, c_i32, ctypes.POINTER(c_char_p)]),
            "sdag_plan_describe": (c_char_p, [P]),
            "sdag_plan_kernel_name": (S, [P, c_i32, ctypes.POINTER(c_char_p)]),
            "sdag_plan_destroy": (None, [P]),
            "sdag_apply": (S, [P, ctypes.POINTER(c_void_p), c_i32, ctypes.POINTER(c_void_p), c_i32, c_dblp, c_i32,
                               P]),
            "sdag_apply_batched": (S, [P, c_i32, ctypes.POINTER(c_void_p), c_i32, ctypes.POINTER(c_void_p), c_i32,
                                       c_dblp, c_i32, P]),
            "sdag_apply_iterated": (S, [P, c_void_p, c_void_p, c_i32, c_dblp, c_i32, P]),
            "sdag_apply_host": (S, [P, ctypes.POINTER(c_void_p), c_i32, ctypes.POINTER(c_void_p), c_i32, c_dblp,
                                    c_i32, P, c_i64p, c_i64p]),
            "sdag_program_create": (S, [c_char_p, c_i64p, ctypes.POINTER(PlanOpts), ctypes.POINTER(P)]),
            "sdag_program_info": (S, [P, ctypes.POINTER(c_i32), ctypes.POINTER(c_i32), ctypes.POINTER(c_i32),
                                      ctypes.POINTER(c_i32)]),
            "sdag_program_arg": (S, [P, c_i32, c_i32, ctypes.POINTER(c_char_p), ctypes.POINTER(c_i32)]),
            "sdag_program_stage": (S, [P, c_i32, ctypes.POINTER(P)]),
            "sdag_program_apply": (S, [P, c_i32, ctypes.POINTER(c_void_p), c_i32, ctypes.POINTER(c_void_p), c_i32,
                                       c_dblp, c_i32, P]),
            "sdag_program_destroy": (None, [P]),
            "sdag_fusion_schedule": (S, [c_dblp, c_i32, c_i32, ctypes.POINTER(c_i32), c_i32,
                                         ctypes.POINTER(c_i32), c_dblp]),
            "sdag_slab_partition": (S, [c_i64, c_i32, c_i32, c_i32, c_i64p]),
            "sdag_slab_halo": (S, [c_i64, c_i32, c_i32, c_i32, c_i64p]),
            "sdag_slab_partition2": (S, [c_i64, c_i32, c_i32, c_i32, c_i32, c_i64p]),
            "sdag_slab_halo2": (S, [c_i64, c_i32, c_i32, c_i32, c_i32, c_i32, c_i64p]),
            "sdag_nccl_get_unique_id": (S, [ctypes.c_char_p]),
            "sdag_nccl_comm_create": (S, [ctypes.c_char_p, c_i32, c_i32, c_i32, ctypes.POINTER(c_void_p)]),
            "sdag_nccl_comm_destroy": (None, [c_void_p]),
            "sdag_nccl_sendrecv": (S, [c_void_p, c_i32, c_void_p, c_void_p, ctypes.c_int64, c_void_p]),
            "sdag_dist_create": (S, [c_char_p, c_i64p, ctypes.POINTER(PlanOpts), c_i32, c_i32, c_void_p,
                                     ctypes.POINTER(P)]),
            "sdag_dist_layout": (S, [P, c_i64p, c_i64p]),
            "sdag_dist_create_local": (S, [P, c_i32, c_i32, c_void_p, c_i32, ctypes.POINTER(P)]),
            "sdag_dist_alloc_dims": (S, [P, c_i64p, c_i64p]),
            "sdag_dist_local_plan": (P, [P]),
            "sdag_dist_apply": (S, [P, ctypes.POINTER(c_void_p), c_i32, ctypes.POINTER(c_void_p), c_i32, c_dblp,
                                    c_i32, P, P]),
            "sdag_dist_apply_iterated": (S, [P, c_void_p, c_void_p, c_i32, c_dblp, c_i32, P, P]),
            "sdag_dist_apply_iterated_loopback": (S, [ctypes.POINTER(P), c_i32, ctypes.POINTER(c_void_p),
                                                      ctypes.POINTER(c_void_p), c_i32, c_dblp, c_i32, P]),
            "sdag_dist_destroy": (None, [P]),
            "sdag_dist_apply_host": (S, [P, ctypes.POINTER(c_void_p), c_i32, ctypes.POINTER(c_void_p), c_i32, c_dblp,
                                         c_i32, P, c_i64p, c_i64p]),
            "sdag_spec_fission": (S, [c_char_p, c_i32, ctypes.c_char_p, c_i64, c_i64p]),
            "sdag_program_fuse": (S, [c_char_p, c_i32, ctypes.c_char_p, c_i64, c_i64p]),
            "sdag_program_version": (S, [c_char_p, c_i32, ctypes.POINTER(c_i32), c_i32, ctypes.c_char_p, c_i64,
                                         c_i64p]),
            "sdag_program_forest": (S, [c_char_p, c_i32, ctypes.POINTER(c_i32), ctypes.POINTER(c_i32),
                                        ctypes.POINTER(c_i32)]),
            "sdag_program_forest_tune": (S, [c_char_p, c_i64p, ctypes.POINTER(PlanOpts), ctypes.POINTER(c_void_p),
                                             c_i32, ctypes.POINTER(c_void_p), c_i32, c_dblp, c_i32, P, c_i32,
                                             c_dblp, ctypes.POINTER(c_i32), ctypes.POINTER(c_i32)]),
            "sdag_plan_profile": (S, [P, ctypes.POINTER(c_void_p), c_i32, ctypes.POINTER(c_void_p), c_i32, c_dblp,
                                      c_i32, ctypes.c_double, ctypes.c_double, P, ctypes.c_void_p]),
            "sdag_dist_p2p_alloc": (S, [P, ctypes.POINTER(c_void_p), ctypes.POINTER(c_void_p)]),
            "sdag_dist_p2p_handle": (S, [P, ctypes.c_char_p]),
            "sdag_dist_p2p_attach": (S, [P, c_i32, ctypes.c_char_p]),
            "sdag_dist_p2p_attach_local": (S, [P, c_i32, P]),
            "sdag_dist_p2p_apply_iterated": (S, [P, c_i32, c_dblp, c_i32, P]),
            "sdag_last_error": (c_char_p, []),
            "sdag_version": (c_char_p, []),
            "sdag_launch_count": (c_i64, []),
            "sdag_measure_fp64_peak": (S, [c_dblp, P]),
            "sdag_registry_count": (c_i32, []),
            "sdag_registry_get": (S, [c_i32, ctypes.POINTER(c_char_p), ctypes.POINTER(c_char_p)]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


class Profile(ctypes.Structure):
    """sdag_profile (include/sdag.h)"""
    _fields_ = [("variant", ctypes.c_char * 96), ("ms", ctypes.c_double), ("flops", ctypes.c_double),
                ("bytes", ctypes.c_double), ("oi_dram", ctypes.c_double), ("ridge", ctypes.c_double),
                ("peak_hbm_gbs", ctypes.c_double), ("peak_fp64_tflops", ctypes.c_double),
                ("frac_dram", ctypes.c_double), ("frac_fp64", ctypes.c_double),
                ("ms_diff_mem", ctypes.c_double), ("ms_diff_arith", ctypes.c_double),
                ("regs", ctypes.c_int32), ("spill_bytes", ctypes.c_int32), ("ctas_per_sm", ctypes.c_int32),
                ("warps_per_sm", ctypes.c_int32), ("bound", ctypes.c_int32), ("hints", ctypes.c_char * 1024)]


# every symbol include/sdag.h declares (checked by tests/test_capi_symbols.py)
EXPORTED = [
    "sdag_plan_opts_init", "sdag_plan_create", "sdag_plan_info_get", "sdag_plan_arg", "sdag_plan_variant_name", "sdag_plan_kernel_name",
    "sdag_plan_describe", "sdag_plan_destroy", "sdag_apply", "sdag_apply_batched", "sdag_apply_iterated",
    "sdag_program_create", "sdag_program_info", "sdag_program_arg", "sdag_program_stage", "sdag_program_apply",
    "sdag_program_destroy",
    "sdag_apply_host", "sdag_fusion_schedule", "sdag_slab_partition", "sdag_slab_halo",
    "sdag_slab_partition2", "sdag_slab_halo2", "sdag_nccl_get_unique_id", "sdag_nccl_comm_create",
    "sdag_nccl_comm_destroy", "sdag_nccl_sendrecv", "sdag_dist_create", "sdag_dist_create_local", "sdag_dist_layout", "sdag_dist_alloc_dims", "sdag_dist_local_plan", "sdag_dist_apply",
    "sdag_dist_apply_iterated", "sdag_dist_destroy", "sdag_dist_apply_host", "sdag_dist_apply_iterated_loopback",
    "sdag_spec_fission", "sdag_program_version", "sdag_program_forest", "sdag_program_forest_tune", "sdag_program_fuse", "sdag_plan_profile", "sdag_dist_p2p_alloc", "sdag_dist_p2p_handle", "sdag_dist_p2p_attach", "sdag_dist_p2p_attach_local",
    "sdag_dist_p2p_apply_iterated", "sdag_last_error",
    "sdag_version", "sdag_launch_count", "sdag_measure_fp64_peak", "sdag_registry_count", "sdag_registry_get",
]
