"""ctypes binding of libsomier.so (include/spread.h, include/somier.h).

Argument marshalling only: every step of the path runs in the library's CUDA
kernels. There is no fallback -- if libsomier.so is missing or fails to load,
import raises (build it with `python -m paper_conf_ipps_torresft22_b200.build`
or __graft_entry__.build()).
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# SOMIER_LIB: experiment hook (tools/variants.sh) to load a variant build; default in-tree
LIB_PATH = os.environ.get("SOMIER_LIB") or os.path.join(_HERE, "libsomier.so")

# spread_status
OK, EINVAL, ENODEV, ENOMEM, ECUDA, ENCCL, ENOTSUP, ESTATE = 0, -1, -2, -3, -4, -5, -6, -7
# somier_exchange
EXCHANGE_FUSED, EXCHANGE_COPY, EXCHANGE_NCCL = 0, 1, 2
# somier_math
MATH_EXACT, MATH_FMA = 0, 1
# spread_sched
SCHED_STATIC, SCHED_DYNAMIC = 0, 1
# spread_map_type
MAP_ALLOC, MAP_TO, MAP_FROM, MAP_TOFROM = 0, 1, 2, 3
# somier_kernel
K1_AUTO, K1_DIRECT, K1_MARCH, K1_MARCH2, K1_TB2 = 0, 1, 2, 3, 4
STATS_HISTORY = 126  # SOMIER_STATS_HISTORY (include/somier.h)


class SpreadError(RuntimeError):
    def __init__(self, status: int, where: str, message: str):
        super().__init__("%s: %s (%s)" % (where, message, status_string(status)))
        self.status = status


class spread_map(ctypes.Structure):
    _fields_ = [("type", ctypes.c_int), ("lo_halo", ctypes.c_int64), ("hi_halo", ctypes.c_int64)]


class somier_params(ctypes.Structure):
    _fields_ = [
        ("n", ctypes.c_int64 * 3),
        ("spacing", ctypes.c_double),
        ("rest_len", ctypes.c_double),
        ("k_spring", ctypes.c_double),
        ("mass", ctypes.c_double),
        ("dt", ctypes.c_double),
        ("amplitude", ctypes.c_double),
        ("seed", ctypes.c_uint64),
        ("kernel", ctypes.c_int32),
        ("exchange", ctypes.c_int32),
        ("math", ctypes.c_int32),
        ("reserved", ctypes.c_int32),
    ]


class somier_stats_t(ctypes.Structure):
    _fields_ = [
        ("step", ctypes.c_int64),
        ("centre", ctypes.c_double * 3),
        ("vmax", ctypes.c_double),
        ("sum_lo", ctypes.c_uint64 * 3),
        ("sum_hi", ctypes.c_int64 * 3),
        ("vmax2_bits", ctypes.c_uint64),
        ("nodes", ctypes.c_int64),
    ]


class somier_timing_t(ctypes.Structure):
    _fields_ = [
        ("launches", ctypes.c_int64),
        ("wait_ms", ctypes.c_double),
        ("kernel_ms", ctypes.c_double),
        ("wait_max_ms", ctypes.c_double),
        ("kernel_max_ms", ctypes.c_double),
    ]


class spread_task_record(ctypes.Structure):
    _fields_ = [("chunk", ctypes.c_int64), ("kind", ctypes.c_int32), ("pad", ctypes.c_int32),
                ("start_ms", ctypes.c_double), ("end_ms", ctypes.c_double)]


class spread_reduce_result(ctypes.Structure):
    _fields_ = [
        ("value", ctypes.c_double),
        ("sum_lo", ctypes.c_uint64),
        ("sum_hi", ctypes.c_int64),
        ("count", ctypes.c_int64),
    ]


REDUCE_SUM, REDUCE_MIN, REDUCE_MAX = 0, 1, 2

_lib = None

# (name, restype, argtypes): every symbol include/*.h declares.
_I64P = ctypes.POINTER(ctypes.c_int64)
_IP = ctypes.POINTER(ctypes.c_int)
_VP = ctypes.c_void_p
_DP = ctypes.POINTER(ctypes.c_double)
SIGNATURES = [
    ("spread_create", ctypes.c_int, [_IP, ctypes.c_int, ctypes.c_int64, ctypes.c_int64, ctypes.c_int, ctypes.c_int64,
                                     ctypes.POINTER(_VP)]),
    ("spread_create_sizes", ctypes.c_int, [_IP, ctypes.c_int, ctypes.c_int64, ctypes.c_int64, _I64P, ctypes.c_int64,
                                           ctypes.POINTER(_VP)]),
    ("spread_create_weighted", ctypes.c_int, [_IP, ctypes.c_int, ctypes.c_int64, ctypes.c_int64, _DP,
                                              ctypes.POINTER(_VP)]),
    ("spread_destroy", ctypes.c_int, [_VP]),
    ("spread_num_chunks", ctypes.c_int, [_VP, _I64P]),
    ("spread_num_devices", ctypes.c_int, [_VP, _IP]),
    ("spread_device", ctypes.c_int, [_VP, ctypes.c_int, _IP]),
    ("spread_chunk_size", ctypes.c_int, [_VP, _I64P]),
    ("spread_range", ctypes.c_int, [_VP, _I64P, _I64P]),
    ("spread_get_chunk", ctypes.c_int, [_VP, ctypes.c_int64, _IP, _IP, _I64P, _I64P]),
    ("spread_chunk_of", ctypes.c_int, [_VP, ctypes.c_int64, _I64P]),
    ("spread_map_extent", ctypes.c_int, [_VP, ctypes.c_int64, spread_map, ctypes.c_int64, _I64P, _I64P]),
    ("spread_stencil3", ctypes.c_int, [_VP, _DP, _DP, ctypes.c_int64]),
    ("spread_reduce", ctypes.c_int, [_VP, _DP, ctypes.c_int64, ctypes.c_int, ctypes.c_int,
                                     ctypes.POINTER(spread_reduce_result)]),
    ("spread_schedule_kind", ctypes.c_int, [_VP, _IP]),
    ("spread_tasks_create", ctypes.c_int, [_VP, _IP, ctypes.POINTER(_VP)]),
    ("spread_enter_data", ctypes.c_int, [_VP, _DP, ctypes.c_int64, spread_map, ctypes.POINTER(_VP)]),
    ("spread_task_stencil3", ctypes.c_int, [_VP, _VP, _VP]),
    ("spread_task_reduce", ctypes.c_int, [_VP, _VP, ctypes.c_int, ctypes.POINTER(spread_reduce_result)]),
    ("spread_exit_data", ctypes.c_int, [_VP, _VP, _DP]),
    ("spread_taskwait", ctypes.c_int, [_VP]),
    ("spread_tasks_set_trace", ctypes.c_int, [_VP, ctypes.c_int]),
    ("spread_tasks_trace", ctypes.c_int, [_VP, ctypes.POINTER(spread_task_record), ctypes.c_int64, _I64P]),
    ("spread_tasks_destroy", ctypes.c_int, [_VP]),
    ("spread_tasks_hold", ctypes.c_int, [_VP, ctypes.c_int64]),
    ("spread_tasks_release", ctypes.c_int, [_VP]),
    ("spread_last_error", ctypes.c_char_p, []),
    ("spread_status_string", ctypes.c_char_p, [ctypes.c_int]),
    ("somier_init", ctypes.c_int, [_VP, ctypes.POINTER(somier_params), ctypes.POINTER(_VP)]),
    ("somier_init_on", ctypes.c_int, [_VP, ctypes.POINTER(somier_params), _IP, ctypes.POINTER(_VP)]),
    ("somier_init_local", ctypes.c_int, [_VP, ctypes.POINTER(somier_params), ctypes.c_int, ctypes.c_int,
                                         ctypes.POINTER(_VP)]),
    ("somier_ipc_export", ctypes.c_int, [_VP, _VP, ctypes.c_size_t, ctypes.POINTER(ctypes.c_size_t)]),
    ("somier_ipc_connect", ctypes.c_int, [_VP, ctypes.POINTER(_VP), ctypes.POINTER(ctypes.c_size_t), ctypes.c_int]),
    ("somier_step", ctypes.c_int, [_VP, ctypes.c_int64]),
    ("somier_sync", ctypes.c_int, [_VP]),
    ("somier_stats", ctypes.c_int, [_VP, ctypes.POINTER(somier_stats_t)]),
    ("somier_stats_history", ctypes.c_int, [_VP, ctypes.c_int64, ctypes.c_int64, ctypes.POINTER(somier_stats_t)]),
    ("somier_set_timing", ctypes.c_int, [_VP, ctypes.c_int]),
    ("somier_nccl_unique_id", ctypes.c_int, [_VP]),
    ("somier_nccl_connect", ctypes.c_int, [_VP, _VP, ctypes.c_int]),
    ("somier_take_timing", ctypes.c_int, [_VP, ctypes.POINTER(somier_timing_t)]),
    ("somier_stats_combine", ctypes.c_int, [ctypes.POINTER(somier_stats_t), ctypes.c_int,
                                            ctypes.POINTER(somier_params), ctypes.POINTER(somier_stats_t)]),
    ("somier_read", ctypes.c_int, [_VP] + [_DP] * 6),
    ("somier_read_planes", ctypes.c_int, [_VP, ctypes.c_int64, ctypes.c_int64] + [_DP] * 6),
    ("somier_load", ctypes.c_int, [_VP] + [_DP] * 6),
    ("somier_set_stream", ctypes.c_int, [_VP, ctypes.c_int, _VP]),
    ("somier_get_stream", ctypes.c_int, [_VP, ctypes.c_int, ctypes.POINTER(_VP)]),
    ("somier_step_count", ctypes.c_int, [_VP, _I64P]),
    ("somier_local_chunks", ctypes.c_int, [_VP, _I64P]),
    ("somier_launch_count", ctypes.c_int, [_VP, _I64P]),
    ("somier_device_bytes", ctypes.c_int, [_VP, _I64P]),
    ("somier_kernel_in_use", ctypes.c_int, [_VP, ctypes.POINTER(ctypes.c_int32)]),
    ("somier_destroy", ctypes.c_int, [_VP]),
    ("somier_version", ctypes.c_char_p, []),
    ("somier_stream_create", ctypes.c_int, [_VP, ctypes.POINTER(somier_params), ctypes.c_int, ctypes.POINTER(_VP)]),
    ("somier_stream_create_on", ctypes.c_int, [_VP, ctypes.POINTER(somier_params), ctypes.c_int, _IP,
                                               ctypes.POINTER(_VP)]),
    ("somier_stream_generate", ctypes.c_int, [_VP] + [_DP] * 6),
    ("somier_stream_step", ctypes.c_int, [_VP] + [_DP] * 9 + [ctypes.POINTER(somier_stats_t)]),
    ("somier_stream_run", ctypes.c_int, [_VP] + [_DP] * 9 + [ctypes.c_int64, ctypes.POINTER(somier_stats_t)]),
    ("somier_stream_traffic", ctypes.c_int, [_VP, _I64P, _I64P, _I64P]),
    ("somier_stream_run2", ctypes.c_int, [_VP] + [_DP] * 12 + [ctypes.c_int64, ctypes.POINTER(somier_stats_t)]),
    ("somier_stream_traffic2", ctypes.c_int, [_VP, _I64P, _I64P]),
    ("somier_stream_run_blocked", ctypes.c_int,
     [_VP] + [_DP] * 12 + [ctypes.c_int64, ctypes.c_int64, ctypes.POINTER(somier_stats_t)]),
    ("somier_stream_traffic_blocked", ctypes.c_int, [_VP, ctypes.c_int64, _I64P, _I64P]),
    ("somier_stream_chunk_counts", ctypes.c_int, [_VP, _I64P]),
    ("somier_stream_set_delay", ctypes.c_int, [_VP, ctypes.c_int, ctypes.c_int64]),
    ("somier_stream_destroy", ctypes.c_int, [_VP]),
]


def _default_nccl() -> None:
    """SOMIER_EXCHANGE_NCCL loads NCCL at run time (SOMIER_NCCL_LIB): default to
    the libnccl.so.2 torch.distributed itself uses, so one NCCL serves both."""
    if os.environ.get("SOMIER_NCCL_LIB"):
        return
    try:
        import nvidia.nccl  # the wheel torch's NCCL backend loads

        path = os.path.join(list(nvidia.nccl.__path__)[0], "lib", "libnccl.so.2")
        if os.path.exists(path):
            os.environ["SOMIER_NCCL_LIB"] = path
    except Exception:
        pass


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError("libsomier.so not built at %s: run __graft_entry__.build() "
                              "(there is no CPU fallback)" % LIB_PATH)
        _default_nccl()
        L = ctypes.CDLL(LIB_PATH)
        for name, res, args in SIGNATURES:
            fn = getattr(L, name)
            fn.restype = res
            fn.argtypes = args
        _lib = L
    return _lib


def status_string(st: int) -> str:
    return lib().spread_status_string(st).decode()


def check(st: int, where: str) -> None:
    if st != OK:
        raise SpreadError(st, where, lib().spread_last_error().decode())
