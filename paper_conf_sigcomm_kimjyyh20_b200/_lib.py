"""ctypes binding of libsr.so (include/sr.h).  Argument marshalling only: every step of the hot path runs
in the library's CUDA kernels.  There is no CPU fallback: if libsr.so is missing or CUDA is unavailable,
loading raises."""
from __future__ import annotations

import ctypes as C
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libsr.so")

SR_OK, SR_E_INVAL, SR_E_NOMEM, SR_E_CUDA, SR_E_NCCL, SR_E_STATE, SR_E_UNSUPPORTED = 0, -1, -2, -3, -4, -5, -6
SR_TRAIN, SR_SERVE, SR_PREV, SR_INIT, SR_BILINEAR = 0, 1, 2, 3, 4
MODELS = {"train": SR_TRAIN, "serve": SR_SERVE, "prev": SR_PREV, "init": SR_INIT, "bilinear": SR_BILINEAR}


class sr_options(C.Structure):
    _fields_ = [("seed", C.c_uint64), ("lr", C.c_float), ("beta1", C.c_float), ("beta2", C.c_float),
                ("eps", C.c_float), ("recent_k", C.c_int), ("recent_w", C.c_int), ("world", C.c_int),
                ("rank", C.c_int), ("dp_weight", C.c_float), ("pool_capacity", C.c_int), ("loss", C.c_int),
                ("skip", C.c_int), ("device", C.c_int), ("nccl_id", C.c_void_p)]


class sr_quality(C.Structure):
    _fields_ = [("psnr_a", C.c_double), ("psnr_b", C.c_double), ("gain", C.c_double)]


class sr_controller(C.Structure):
    _fields_ = [("thresh_sat", C.c_double), ("count_sat", C.c_int), ("thresh_online", C.c_double),
                ("count_online", C.c_int), ("state", C.c_int), ("patience", C.c_int)]


class sr_epoch_report(C.Structure):
    _fields_ = [("state_before", C.c_int), ("event", C.c_int), ("state_after", C.c_int), ("diff", C.c_double),
                ("psnr_serve", C.c_double), ("psnr_prev", C.c_double), ("psnr_init", C.c_double),
                ("psnr_bilinear", C.c_double), ("q_dnn", C.c_double), ("q_dnn_prev", C.c_double)]


SR_TRAINING, SR_SUSPENDED = 0, 1
SR_EV_NONE, SR_EV_SUSPEND, SR_EV_RESUME = 0, 1, 2

_P = C.c_void_p
_I = C.c_int
_SIGS = {
    "sr_create": (_I, [_I, _I, _I, C.POINTER(sr_options), C.POINTER(_P)]),
    "sr_destroy": (None, [_P]),
    "sr_last_error": (C.c_char_p, [_P]),
    "sr_num_params": (C.c_size_t, [_P]),
    "sr_get_params": (_I, [_P, _I, _P, C.c_size_t]),
    "sr_set_params": (_I, [_P, _P, C.c_size_t]),
    "sr_infer": (_I, [_P, _I, _P, _I, _I, _I, _P, _P]),
    "sr_infer_host": (_I, [_P, _I, _P, _I, _I, _I, _P, _P]),
    "sr_infer_host_async": (_I, [_P, _I, _P, _I, _I, _I, _P, _P]),
    "sr_infer_host_wait": (_I, [_P]),
    "sr_infer_rows": (_I, [_P, _I, _P, _I, _I, _I, _I, _P, _P]),
    "sr_infer_i420": (_I, [_P, _I, _P, _P, _P, _I, _I, _I, _P, _P, _P, _P]),
    "sr_pool_push_i420": (_I, [_P, _P, _P, _P, _I, _I, _P, _P, _I, _I, _P, _P]),
    "sr_train_step": (_I, [_P, _P, _P, _I, _I, _P, _P]),
    "sr_train_grad": (_I, [_P, _P, _P, _I, _I, _P, _P]),
    "sr_grad_buffer": (_P, [_P]),
    "sr_train_apply": (_I, [_P, C.c_float, _P]),
    "sr_train_apply_dev": (_I, [_P, _P, _P]),
    "sr_train_allreduce": (_I, [_P, _P]),
    "sr_dp_weight_sum": (C.c_double, [_P]),
    "sr_nccl_unique_id": (_I, [_P, C.c_size_t]),
    "sr_get_adam_state": (_I, [_P, _P, _P, C.c_size_t, C.POINTER(C.c_int64)]),
    "sr_pool_stats": (_I, [_P, C.POINTER(C.c_int64), C.POINTER(C.c_int64)]),
    "sr_pool_push": (_I, [_P, _P, _P, _I, _I, _P, _P]),
    "sr_pool_size": (C.c_size_t, [_P]),
    "sr_sample_batch": (_I, [_P, C.c_int64, _I, _I, _P, _P, _P, _P]),
    "sr_train_sampled": (_I, [_P, _I, _I, _I, _P, _P]),
    "sr_publish": (_I, [_P, _P]),
    "sr_psnr_gain": (_I, [_P, _I, _I, _P, _P, _I, _I, C.POINTER(sr_quality), _P]),
    "sr_controller_init": (_I, [C.POINTER(sr_controller), C.c_double, _I, C.c_double, _I]),
    "sr_controller_update": (_I, [C.POINTER(sr_controller), C.c_double, C.POINTER(_I)]),
    "sr_controller_step": (_I, [_P, C.POINTER(sr_controller), _P, _P, _I, _I, C.POINTER(sr_epoch_report), _P]),
    "sr_patch_select": (_I, [_P, _P, _P, _I, _I, _I, _I, C.c_uint64, C.c_int64, _P, C.POINTER(_I), _P]),
    "sr_sse_u8": (_I, [_P, _P, _I, C.c_int64, _P, _P]),
    "sr_launch_count": (C.c_uint64, [_P]),
    "sr_kernel_timing": (_I, [_P, _I]),
    "sr_set_fusion": (_I, [_P, _I]),
    "sr_set_sm_split": (_I, [_P, _I]),
    "sr_sm_partition": (_I, [_I, C.POINTER(_P), C.POINTER(_P), C.POINTER(_I), C.POINTER(_I)]),
    "sr_sm_partition_release": (_I, []),
    "sr_kernel_stats": (_I, [_P, C.c_char_p, C.c_size_t]),
    "sr_test_pack_input": (_I, [_P, _I, _I, _I, _P, _P]),
    "sr_test_conv": (_I, [_P, _I, _I, _I, _I, _I, _P, _P, _P, _P, _I, _I, _P, _P]),
    "sr_test_wgrad": (_I, [_P, _P, _I, _I, _I, _I, _I, _P, _P, _P]),
    "sr_test_wgrad_batch": (_I, [_I, _P, _P, _I, _I, _I, _P, _P, _P, _P]),
    "sr_test_adam": (_I, [_P, _P, _P, _P, C.c_size_t, _I, C.c_float, _P]),
    "sr_test_mma2": (_I, [_P, _P, _P, _I, _I, _P]),
    "sr_test_mma": (_I, [_P, _P, _P, _I, _I, _I, _I, _I, _I, _P, _P]),
    "sr_test_tma": (_I, [_P, _I, _I, _I, _I, _I, _I, _I, _I, _I, _I, _P, _P]),
}

_lib = None


def load(path: str = LIB_PATH):
    """Load libsr.so and bind every exported call; raises if it is missing (no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise RuntimeError(f"libsr.so not built at {path}: run `python -m paper_conf_sigcomm_kimjyyh20_b200.build`")
    lib = C.CDLL(path)
    for name, (res, args) in _SIGS.items():
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    _lib = lib
    return lib


class SRError(RuntimeError):
    pass


def check(status: int, ctx=None, what: str = ""):
    if status != SR_OK:
        msg = ""
        if ctx is not None:
            m = load().sr_last_error(ctx)
            msg = m.decode() if m else ""
        raise SRError(f"{what} failed with status {status}: {msg}")
