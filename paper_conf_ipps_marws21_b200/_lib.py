"""ctypes declarations of libhogbatch.so (include/hogbatch.h).  Argument marshalling only.

The library is the in-tree ``libhogbatch.so`` built by ``build.py`` (sm_100a).  There is no
fallback: if the library is missing or cannot be loaded, importing this module raises.
"""
from __future__ import annotations

import ctypes as C
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("HB_LIB") or os.path.join(HERE, "libhogbatch.so")  # HB_LIB: A/B builds

HB_OK, HB_EINVAL, HB_ENOMEM, HB_ECUDA, HB_ENCCL, HB_ESTATE, HB_EUNSUPPORTED = 0, -1, -2, -3, -4, -5, -6
HB_SIGMOID = 0
HB_PREC_BF16, HB_PREC_FP32_CHECK = 0, 1
HB_BF16, HB_F32 = 0, 1
HB_MINIBATCH, HB_HOGBATCH, HB_STATIC, HB_ADAPTIVE = 0, 1, 2, 3
HB_RESET_FASTEST, HB_RESET_NONE = 0, 1
HB_CREDIT_DISPATCH, HB_CREDIT_COMPLETION = 0, 1
HB_UPDATE_HOGWILD, HB_UPDATE_ATOMIC = 0, 1
# mlp_set_option keys
OPTIONS = {"fused_min_batch": 0, "rowchain": 1, "rc_cluster": 2, "bwd_overlap": 3, "head_fuse": 4, "dw_pair": 5,
           "pdl": 6, "graphs": 7, "inflight": 8, "stage_rows": 9, "update": 10, "step_kernel_max_b": 11,
           "gemm_pair": 12, "head_kernel": 13}
ACTIONS = ("none", "halve", "double", "clamp_lo", "clamp_hi")

# every symbol include/hogbatch.h declares (checked by tests/test_abi.py)
EXPORTS = ("hb_last_error", "hb_abi_version", "hb_device_ok", "mlp_create", "mlp_destroy",
           "mlp_num_params", "mlp_fused_path", "mlp_set_option", "mlp_get_option", "mlp_get_params",
           "mlp_set_params", "mlp_worker_create", "mlp_worker_params", "mlp_worker_destroy", "mlp_worker_stream",
           "mlp_step", "mlp_step_grads", "mlp_row_losses", "mlp_loss", "hb_schedule_trace", "hogbatch_run",
           "hb_nccl_unique_id", "hb_comm_create", "hb_comm_destroy", "hb_merge_begin", "hb_merge",
           "hb_merge_replicas", "hb_kernel_launches", "hb_prof_enable", "hb_prof_read", "hb_merge_schedule",
           "mlp_worker_create_nested", "hb_coord_create", "hb_coord_destroy", "hb_coord_reset",
           "hb_coord_schedule", "hb_coord_idle", "mlp_attach_peers", "mlp_ipc_handle", "mlp_attach_ipc_peers")
# tuning build only (include/hogbatch_tuning.h): not exported by the product library
TUNING_EXPORTS = ("hb_bench_gemm", "hb_bench_gemm_phases", "hb_rc_trace", "hb_bench_step", "hb_bench_sgd_apply")
PROF_LAYERS = 16
PROF_CLASSES = ("fwd_gemm", "head_gemm", "softmax_xent", "dgrad_gemm", "wgrad_sgd_gemm", "bias_sgd", "other",
                "rowchain", "step_kernel", "head_kernel")


class WorkerPolicy(C.Structure):
    _fields_ = [("min_b", C.c_int32), ("max_b", C.c_int32), ("init_b", C.c_int32),
                ("incr", C.c_float), ("c0", C.c_double), ("c1", C.c_double)]


class Policy(C.Structure):
    _fields_ = [("kind", C.c_int32), ("alpha", C.c_int32), ("eta0", C.c_double), ("b0", C.c_int32),
                ("reset", C.c_int32), ("credit", C.c_int32), ("deterministic", C.c_int32),
                ("eval_loss", C.c_int32), ("max_steps", C.c_int64), ("merges_per_epoch", C.c_int32),
                ("merge_gamma", C.c_float), ("comm", C.c_void_p), ("n_workers", C.c_int32),
                ("workers", C.POINTER(WorkerPolicy)), ("update", C.c_int32), ("epoch_barrier", C.c_int32),
                ("check_labels", C.c_int32), ("coord", C.c_void_p), ("first_worker", C.c_int32)]


HB_DATA_DENSE, HB_DATA_CSR = 0, 1


class Dataset(C.Structure):
    _fields_ = [("X", C.c_void_p), ("ldx", C.c_int64), ("x_dtype", C.c_int32),
                ("y", C.c_void_p), ("n", C.c_int64), ("format", C.c_int32), ("n_cols", C.c_int64),
                ("indptr", C.c_void_p), ("indices", C.c_void_p), ("values", C.c_void_p)]


class TraceRec(C.Structure):
    _fields_ = [("seq", C.c_int64), ("epoch", C.c_int32), ("worker", C.c_int32),
                ("vtime", C.c_double), ("u_before", C.c_double),
                ("b_before", C.c_int32), ("action", C.c_int32), ("b_after", C.c_int32),
                ("served", C.c_int32), ("u_after", C.c_double), ("offset", C.c_int64),
                ("lr", C.c_double)]


class Stats(C.Structure):
    _fields_ = [("max_epochs", C.c_int32), ("epochs_done", C.c_int32),
                ("epoch_loss", C.POINTER(C.c_double)), ("epoch_train_s", C.POINTER(C.c_double)),
                ("updates", C.POINTER(C.c_int64)), ("samples", C.POINTER(C.c_int64)),
                ("trace", C.POINTER(TraceRec)), ("trace_cap", C.c_int64), ("trace_len", C.c_int64),
                ("step_loss", C.POINTER(C.c_float)), ("step_loss_cap", C.c_int64),
                ("n_steps", C.c_int64), ("total_train_s", C.c_double),
                ("total_samples", C.c_int64), ("n_merges", C.c_int32), ("want_train_loss", C.c_int32),
                ("train_loss", C.c_double)]


class ProfEntry(C.Structure):
    _fields_ = [("launches", C.c_int64), ("ms", C.c_double), ("flops", C.c_double), ("bytes", C.c_double)]


def load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run `python paper_conf_ipps_marws21_b200/build.py` "
                          "(there is no CPU fallback)")
    lib = C.CDLL(LIB_PATH)
    P, I32, I64, F, D, VP = C.POINTER, C.c_int32, C.c_int64, C.c_float, C.c_double, C.c_void_p
    sig = {
        "hb_last_error": ([], C.c_char_p),
        "hb_abi_version": ([], C.c_int),
        "hb_device_ok": ([I32], C.c_int),
        "mlp_create": ([P(I32), I32, I32, I32, C.c_uint64, I32, P(VP)], C.c_int),
        "mlp_destroy": ([VP], C.c_int),
        "mlp_num_params": ([VP, P(I64)], C.c_int),
        "mlp_fused_path": ([VP, I32, P(I32)], C.c_int),
        "mlp_set_option": ([VP, I32, I64], C.c_int),
        "mlp_get_option": ([VP, I32, P(I64)], C.c_int),
        "mlp_get_params": ([VP, P(F), I64], C.c_int),
        "mlp_set_params": ([VP, P(F), I64], C.c_int),
        "mlp_worker_create": ([VP, I32, I32, I32, VP, P(VP)], C.c_int),
        "mlp_worker_params": ([VP, P(F), I64], C.c_int),
        "mlp_worker_destroy": ([VP], C.c_int),
        "mlp_worker_create_nested": ([VP, I32, I32, VP, P(VP)], C.c_int),
        "mlp_worker_stream": ([VP], VP),
        "mlp_step": ([VP, VP, I64, I32, VP, I32, F, P(F)], C.c_int),
        "mlp_step_grads": ([VP, VP, I64, I32, VP, I32, P(F), I64, P(F)], C.c_int),
        "mlp_loss": ([VP, VP, I64, I32, VP, I64, P(D)], C.c_int),
        "mlp_row_losses": ([VP, P(F), I32], C.c_int),
        "hb_schedule_trace": ([P(Policy), I64, I32, P(TraceRec), I64, P(I64)], C.c_int),
        "hogbatch_run": ([P(VP), I32, P(Policy), P(Dataset), I32, P(Stats)], C.c_int),
        "hb_nccl_unique_id": ([P(C.c_uint8)], C.c_int),
        "hb_comm_create": ([P(C.c_uint8), I32, I32, I32, P(VP)], C.c_int),
        "hb_comm_destroy": ([VP], C.c_int),
        "hb_merge_begin": ([VP], C.c_int),
        "hb_merge": ([VP, VP, F, VP], C.c_int),
        "hb_merge_replicas": ([VP, P(VP), I32, F], C.c_int),
        "mlp_attach_peers": ([VP, P(VP), I32, F], C.c_int),
        "mlp_ipc_handle": ([VP, P(C.c_uint8)], C.c_int),
        "mlp_attach_ipc_peers": ([VP, P(C.c_uint8), I32, F], C.c_int),
        "hb_coord_create": ([C.c_char_p, P(Policy), I64, I32, I32, P(VP)], C.c_int),
        "hb_coord_destroy": ([VP], C.c_int),
        "hb_coord_reset": ([VP, P(Policy), I64], C.c_int),
        "hb_coord_schedule": ([VP, I32, D, P(TraceRec)], C.c_int),
        "hb_coord_idle": ([VP, I32, P(I32)], C.c_int),
        "hb_kernel_launches": ([], I64),
        "hb_prof_enable": ([I32], C.c_int),
        "hb_rc_trace": ([VP, I64], C.c_int),
        "hb_bench_step": ([VP, VP, I64, VP, I32, I32, I32, P(F)], C.c_int),
        "hb_bench_sgd_apply": ([I64, I32, P(F)], C.c_int),
        "hb_prof_read": ([P(ProfEntry), I32, I32], C.c_int),
        "hb_bench_gemm": ([I32, I32, I32, I32, I32, P(F)], C.c_int),
        "hb_bench_gemm_phases": ([I32, I32, I32, I32, P(C.c_uint64), I64], C.c_int),
        "hb_merge_schedule": ([I64, I32, P(I32), I64, P(I32), P(I32)], C.c_int),
    }
    for name, (args, res) in sig.items():
        if (os.environ.get("HB_LIB") or name in TUNING_EXPORTS) and not hasattr(lib, name):
            continue  # tuning entry points exist only in the tuning build; A/B builds may lack new ones
        fn = getattr(lib, name)
        fn.argtypes = args
        fn.restype = res
    return lib


class HogbatchError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"[{code}] {msg}")
        self.code = code
