"""paper_conf_ipps_torresft22_b200 -- B200-native Somier "target spread" step.

The data-parallel hot path of Torres, Ferrer, Teruel (IPDPSW 2022): the Somier
spring-lattice time step (§V) spread over the GPUs of one node with the
paper's spread schedules (§III-B; irregular and dynamic: §IX). C ABI: include/spread.h and
include/somier.h, implemented by libsomier.so (hand-written sm_100a kernels).
This package is the Python binding (argument marshalling only).
"""
from . import _native, capi
from ._native import (EXCHANGE_COPY, EXCHANGE_FUSED, EXCHANGE_NCCL, K1_AUTO, K1_DIRECT, K1_MARCH, K1_MARCH2,
                      K1_TB2, MATH_EXACT, MATH_FMA, SCHED_DYNAMIC, SCHED_STATIC, STATS_HISTORY, SpreadError)
from .somier import Somier, SomierParams, SomierStream, Stats, combine_stats
from .spread import Chunk, Spread, SpreadTasks

__all__ = ["capi", "Spread", "SpreadTasks", "Chunk", "Somier", "SomierParams", "SomierStream", "Stats",
           "combine_stats", "SpreadError", "K1_AUTO", "K1_DIRECT", "K1_MARCH", "K1_MARCH2", "K1_TB2",
           "SCHED_STATIC", "SCHED_DYNAMIC", "EXCHANGE_FUSED", "EXCHANGE_COPY", "EXCHANGE_NCCL", "MATH_EXACT", "MATH_FMA",
           "STATS_HISTORY",
           "version"]


def version() -> str:
    return _native.lib().somier_version().decode()
