"""ctypes binding of liborion (include/orion.h, include/orion_kernels.h): argument marshalling only.

Every step of the hot path runs inside liborion.so (C++ scheduler + sm_100a kernels). There is no
Python or CPU fallback: if the library is missing this module raises at import.
"""
import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liborion.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"liborion.so not built at {LIB_PATH}; run `python -c 'import __graft_entry__ as g; g.build()'`")
lib = ctypes.CDLL(LIB_PATH)

# ---- constants (orion.h)
OK, E_INVAL, E_STATE, E_AGAIN, E_CUDA, E_NOMEM, E_TIMEOUT, E_NODEV = 0, -1, -2, -3, -4, -5, -6, -7
HP, BE = 0, 1
CLS_U, CLS_C, CLS_M = 0, 1, 2
OP_KERNEL, OP_MEMCPY_H2D, OP_MEMCPY_D2H, OP_MEMSET, OP_MEMCPY_D2D = 0, 1, 2, 3, 4
OPF_REQ_BEGIN, OPF_REQ_END = 1, 2
F_HP_BUSY_REQUEST, F_HP_REF_ALL, F_HP_UNKNOWN_STRICT, F_THROTTLE_ONLY_HP_BUSY, F_FREE_SMS = 1, 2, 4, 8, 16
F_NO_PRIORITY, F_NO_PROFILE_TEST, F_NO_SM_TEST, F_NO_THROTTLE = 32, 64, 128, 256
# policy ablation (Fig. 14) and the Streams baselines
POLICIES = {"orion": 0, "orion_noprio": F_NO_PRIORITY, "profiles": F_NO_SM_TEST, "priorities": F_NO_PROFILE_TEST | F_NO_SM_TEST | F_NO_THROTTLE,
            "streams": F_NO_PRIORITY | F_NO_PROFILE_TEST | F_NO_SM_TEST | F_NO_THROTTLE}
BACKEND_CUDA, BACKEND_FAKE = 0, 1
MAX_ARGS = 24
WS_TICKET_BYTES = 65536   # kernels/common.cuh: ticket region at the start of every workspace


class Profile(ctypes.Structure):
    _fields_ = [("kernel_id", ctypes.c_uint32), ("cls", ctypes.c_uint8), ("pad", ctypes.c_uint8 * 3),
                ("sm_needed", ctypes.c_uint32), ("reserved", ctypes.c_uint32), ("dur_ns", ctypes.c_uint64)]


class Op(ctypes.Structure):
    _fields_ = [("fn", ctypes.c_uint32), ("kind", ctypes.c_uint16), ("nargs", ctypes.c_uint8),
                ("opflags", ctypes.c_uint8), ("prof", Profile), ("args", ctypes.c_uint64 * MAX_ARGS)]


class Config(ctypes.Structure):
    _fields_ = [("num_sms", ctypes.c_uint32), ("sm_threshold", ctypes.c_uint32),
                ("dur_threshold_ppm", ctypes.c_uint32), ("be_partition_sms", ctypes.c_uint32),
                ("hp_latency_ns", ctypes.c_uint64), ("flags", ctypes.c_uint32), ("queue_capacity", ctypes.c_uint32),
                ("backend", ctypes.c_uint32), ("sched_cpu", ctypes.c_int32), ("log_capacity", ctypes.c_uint64),
                ("fake_time_scale_pct", ctypes.c_uint32), ("trace_kernel_id_plus1", ctypes.c_uint32),
                ("fake_contention", ctypes.c_uint32), ("reserved", ctypes.c_uint32 * 5)]


class KernelInfo(ctypes.Structure):   # orion_kernel_info_t
    _fields_ = [("grid_ctas", ctypes.c_uint64), ("threads_per_cta", ctypes.c_int32), ("regs_per_thread", ctypes.c_int32),
                ("static_smem", ctypes.c_int32), ("dynamic_smem", ctypes.c_int32), ("blocks_per_sm", ctypes.c_int32),
                ("pipe", ctypes.c_int32), ("kernel", ctypes.c_char * 120), ("launches", ctypes.c_int32)]


PIPE_FMA, PIPE_TF32X3, PIPE_BF16 = 0, 1, 2

assert ctypes.sizeof(Op) == 224 and ctypes.sizeof(Profile) == 24

_h = ctypes.c_void_p
_sig = {
    "orion_create": (ctypes.c_int, [ctypes.c_int, ctypes.POINTER(Config), ctypes.POINTER(_h)]),
    "orion_register_client": (ctypes.c_int, [_h, ctypes.c_int, ctypes.POINTER(ctypes.c_int)]),
    "orion_client_stream": (ctypes.c_int, [_h, ctypes.c_int, ctypes.POINTER(ctypes.c_void_p)]),
    "orion_start": (ctypes.c_int, [_h]),
    "orion_submit": (ctypes.c_int, [_h, ctypes.c_int, ctypes.POINTER(Op), ctypes.POINTER(ctypes.c_uint64)]),
    "orion_submit_n": (ctypes.c_int, [_h, ctypes.c_int, ctypes.POINTER(Op), ctypes.c_uint32, ctypes.POINTER(ctypes.c_uint64)]),
    "orion_synchronize": (ctypes.c_int, [_h, ctypes.c_int, ctypes.c_uint64]),
    "orion_done_seq": (ctypes.c_int, [_h, ctypes.c_int, ctypes.POINTER(ctypes.c_uint64)]),
    "orion_stop": (ctypes.c_int, [_h]),
    "orion_read_log": (ctypes.c_int, [_h, ctypes.c_void_p, ctypes.c_size_t, ctypes.POINTER(ctypes.c_size_t)]),
    "orion_stats": (ctypes.c_int, [_h, ctypes.POINTER(ctypes.c_uint64), ctypes.c_uint32]),
    "orion_destroy": (ctypes.c_int, [_h]),
    "orion_strerror": (ctypes.c_char_p, [ctypes.c_int]),
    "orion_run_requests": (ctypes.c_int, [_h, ctypes.c_int, ctypes.POINTER(Op), ctypes.c_uint32, ctypes.c_void_p,
                                          ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p]),
    "orion_run_requests_direct": (ctypes.c_int, [_h, ctypes.c_int, ctypes.POINTER(Op), ctypes.c_uint32, ctypes.c_void_p,
                                                 ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p]),
    "orion_run_iterations": (ctypes.c_int, [_h, ctypes.c_int, ctypes.POINTER(Op), ctypes.c_uint32, ctypes.c_uint32,
                                            ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_uint64,
                                            ctypes.POINTER(ctypes.c_uint64)]),
    "orion_now_ns": (ctypes.c_int64, []),
    "orion_trace_read": (ctypes.c_int, [_h, ctypes.POINTER(ctypes.c_float), ctypes.c_uint32, ctypes.POINTER(ctypes.c_uint32)]),
    "orion_kernel_count": (ctypes.c_int, []),
    "orion_kernel_name": (ctypes.c_char_p, [ctypes.c_uint32]),
    "orion_kernel_launch": (ctypes.c_int, [ctypes.c_uint32, ctypes.POINTER(ctypes.c_uint64), ctypes.c_uint32, ctypes.c_void_p]),
    "orion_kernel_geometry": (ctypes.c_int, [ctypes.c_uint32, ctypes.POINTER(ctypes.c_uint64), ctypes.c_uint32,
                                             ctypes.POINTER(ctypes.c_uint64), ctypes.POINTER(ctypes.c_int32),
                                             ctypes.POINTER(ctypes.c_int32), ctypes.POINTER(ctypes.c_int32)]),
    "orion_kernel_info": (ctypes.c_int, [ctypes.c_uint32, ctypes.POINTER(ctypes.c_uint64), ctypes.c_uint32,
                                         ctypes.POINTER(KernelInfo)]),
    "orion_gemm_workspace_bytes": (ctypes.c_uint64, [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64]),
    "orion_conv_wgrad_workspace_bytes": (ctypes.c_uint64, [ctypes.c_uint64] * 9),
    "orion_bn_workspace_bytes": (ctypes.c_uint64, [ctypes.c_uint64, ctypes.c_uint64]),
    "orion_layernorm_bwd_workspace_bytes": (ctypes.c_uint64, [ctypes.c_uint64, ctypes.c_uint64]),
    "orion_dw_wgrad_workspace_bytes": (ctypes.c_uint64, [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64]),
}
for _name, (_res, _args) in _sig.items():
    _f = getattr(lib, _name)
    _f.restype = _res
    _f.argtypes = _args

# Exported symbols declared in include/*.h (checked by tests/test_boundary.py)
EXPORTS = sorted(_sig)


class OrionError(RuntimeError):
    def __init__(self, code, what=""):
        self.code = code
        super().__init__(f"{what}: {lib.orion_strerror(code).decode()} ({code})")


def check(code, what=""):
    if code != OK:
        raise OrionError(code, what)
    return code


def kernel_names():
    return [lib.orion_kernel_name(i).decode() for i in range(lib.orion_kernel_count())]


FN = {n: i for i, n in enumerate(kernel_names())}
