"""The `target spread` descriptor (include/spread.h)."""
from __future__ import annotations

import ctypes
from typing import List, NamedTuple, Optional, Sequence

from . import _native as N


class Chunk(NamedTuple):
    index: int
    device_pos: int   # list position: distribution order
    device_id: int
    start: int        # omp_spread_start
    size: int         # omp_spread_size


class Spread:
    """devices(...) + range(start:len) + spread_schedule(static, chunk).

    chunk == 0 means ceil(len / ndevices): one contiguous slab per device.
    Irregular static schedules: Spread.with_sizes / Spread.weighted.
    """

    def __init__(self, devices: Sequence[int], range_start: int, range_len: int, chunk: int = 0, sched: int = 0,
                 *, sizes: Sequence[int] | None = None, weights: Sequence[float] | None = None):
        L = N.lib()
        arr = (ctypes.c_int * len(devices))(*devices)
        h = ctypes.c_void_p()
        if sizes is not None:
            sz = (ctypes.c_int64 * max(1, len(sizes)))(*sizes)
            N.check(L.spread_create_sizes(arr, len(devices), range_start, range_len, sz, len(sizes),
                                          ctypes.byref(h)), "spread_create_sizes")
        elif weights is not None:
            if len(weights) != len(devices):
                raise ValueError("one weight per device")
            w = (ctypes.c_double * len(weights))(*weights)
            N.check(L.spread_create_weighted(arr, len(devices), range_start, range_len, w, ctypes.byref(h)),
                    "spread_create_weighted")
        else:
            N.check(L.spread_create(arr, len(devices), range_start, range_len, sched, chunk, ctypes.byref(h)),
                    "spread_create")
        self._h = h
        self.devices = list(devices)

    @classmethod
    def with_sizes(cls, devices: Sequence[int], range_start: int, range_len: int, sizes: Sequence[int]) -> "Spread":
        """spread_create_sizes: chunk c = the next sizes[c] iterations, on list position c mod p."""
        return cls(devices, range_start, range_len, sizes=sizes)

    @classmethod
    def weighted(cls, devices: Sequence[int], range_start: int, range_len: int, weights: Sequence[float]) -> "Spread":
        """spread_create_weighted: one chunk per device, sized by largest remainder of the weights."""
        return cls(devices, range_start, range_len, weights=weights)

    @property
    def handle(self) -> ctypes.c_void_p:
        return self._h

    def close(self) -> None:
        if self._h:
            N.lib().spread_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    @property
    def num_chunks(self) -> int:
        v = ctypes.c_int64()
        N.check(N.lib().spread_num_chunks(self._h, ctypes.byref(v)), "spread_num_chunks")
        return v.value

    @property
    def chunk_size(self) -> int:
        v = ctypes.c_int64()
        N.check(N.lib().spread_chunk_size(self._h, ctypes.byref(v)), "spread_chunk_size")
        return v.value

    @property
    def range(self):
        a, b = ctypes.c_int64(), ctypes.c_int64()
        N.check(N.lib().spread_range(self._h, ctypes.byref(a), ctypes.byref(b)), "spread_range")
        return a.value, b.value

    def chunk(self, c: int) -> Chunk:
        pos, dev = ctypes.c_int(), ctypes.c_int()
        start, size = ctypes.c_int64(), ctypes.c_int64()
        N.check(N.lib().spread_get_chunk(self._h, c, ctypes.byref(pos), ctypes.byref(dev), ctypes.byref(start),
                                         ctypes.byref(size)), "spread_get_chunk")
        return Chunk(c, pos.value, dev.value, start.value, size.value)

    def chunks(self) -> List[Chunk]:
        return [self.chunk(c) for c in range(self.num_chunks)]

    @property
    def dynamic(self) -> bool:
        """spread_schedule(dynamic, chunk): positions chosen at run time."""
        v = ctypes.c_int()
        N.check(N.lib().spread_schedule_kind(self._h, ctypes.byref(v)), "spread_schedule_kind")
        return v.value == N.SCHED_DYNAMIC

    def chunk_of(self, iteration: int) -> int:
        v = ctypes.c_int64()
        N.check(N.lib().spread_chunk_of(self._h, iteration, ctypes.byref(v)), "spread_chunk_of")
        return v.value

    def stencil3(self, A, B=None):
        """Listing 3: B[i] = A[i-1] + A[i] + A[i+1] over the spread's range, each
        chunk computed on its device (spread_stencil3). Returns B."""
        import numpy as np

        A = np.ascontiguousarray(A, dtype=np.float64)
        B = np.zeros_like(A) if B is None else B
        dp = ctypes.POINTER(ctypes.c_double)
        N.check(N.lib().spread_stencil3(self._h, A.ctypes.data_as(dp), B.ctypes.data_as(dp), A.size),
                "spread_stencil3")
        return B

    def reduce(self, A, op: str = "sum", scale_exp: int = 60):
        """`map(to: A[start:size]) reduction(op: r)` over the spread's range, each
        chunk reduced on its device (spread_reduce). op "sum": the exact
        fixed-point sum S of round_half_even(A[i] * 2^scale_exp) (returned as
        the int S and value = S * 2^-scale_exp); "min" / "max": the extreme
        element (-0 < +0, NaN if any). Returns (value, S or None, count)."""
        import numpy as np

        A = np.ascontiguousarray(A, dtype=np.float64)
        code = {"sum": N.REDUCE_SUM, "min": N.REDUCE_MIN, "max": N.REDUCE_MAX}[op]
        r = N.spread_reduce_result()
        N.check(N.lib().spread_reduce(self._h, A.ctypes.data_as(ctypes.POINTER(ctypes.c_double)), A.size, code,
                                      int(scale_exp), ctypes.byref(r)), "spread_reduce")
        S = (r.sum_hi << 64) + r.sum_lo if op == "sum" else None
        return r.value, S, r.count

    def map_extent(self, c: int, array_len: int, lo_halo: int = 0, hi_halo: int = 0, map_type: int = N.MAP_TO):
        """Section [first, first+len) of A[omp_spread_start-lo : omp_spread_size+lo+hi]."""
        first, ln = ctypes.c_int64(), ctypes.c_int64()
        m = N.spread_map(map_type, lo_halo, hi_halo)
        N.check(N.lib().spread_map_extent(self._h, c, m, array_len, ctypes.byref(first), ctypes.byref(ln)),
                "spread_map_extent")
        return first.value, ln.value


class SpreadTasks:
    """Chunk-level `depend` between spread constructs (include/spread.h,
    PAPER.md:746-767): every method enqueues per chunk and returns (nowait);
    taskwait() is the only barrier. Host arrays passed to enter / exit must stay
    alive (and unchanged / unread) until the next taskwait()."""

    KINDS = {0: "enter", 1: "stencil3", 2: "reduce", 3: "exit"}

    def __init__(self, spread: Spread, cuda_devices: Optional[Sequence[int]] = None):
        self.spread = spread
        h = ctypes.c_void_p()
        arr = None if cuda_devices is None else (ctypes.c_int * len(cuda_devices))(*cuda_devices)
        N.check(N.lib().spread_tasks_create(spread.handle, arr, ctypes.byref(h)), "spread_tasks_create")
        self._h = h
        self._keep = []      # host arrays in flight
        self._results = []   # (spread_reduce_result, [value slot])

    def close(self) -> None:
        if getattr(self, "_h", None):
            N.lib().spread_tasks_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def enter(self, A=None, n: Optional[int] = None, lo_halo: int = 0, hi_halo: int = 0):
        """target enter data spread map(to: A[start-lo : size+lo+hi]) (A given) or
        map(alloc: ...) (A None, n elements) depend(out: A[start:size]) nowait."""
        import numpy as np

        if A is not None:
            A = np.ascontiguousarray(A, dtype=np.float64)
            self._keep.append(A)
            n = A.size
            ptr = A.ctypes.data_as(ctypes.POINTER(ctypes.c_double))
            m = N.spread_map(N.MAP_TO, lo_halo, hi_halo)
        else:
            ptr = None
            m = N.spread_map(N.MAP_ALLOC, lo_halo, hi_halo)
        d = ctypes.c_void_p()
        N.check(N.lib().spread_enter_data(self._h, ptr, int(n), m, ctypes.byref(d)), "spread_enter_data")
        return d

    def stencil3(self, a, b) -> None:
        """target spread depend(in: A[start-1:size+2]) depend(out: B[start:size]) nowait: B[i] = A[i-1]+A[i]+A[i+1]."""
        N.check(N.lib().spread_task_stencil3(self._h, a, b), "spread_task_stencil3")

    def reduce_sum(self, a, scale_exp: int = 60):
        """target spread depend(in: A[start:size]) reduction(+) nowait (exact sum);
        returns a result object, filled by the next taskwait()."""
        r = N.spread_reduce_result()
        N.check(N.lib().spread_task_reduce(self._h, a, int(scale_exp), ctypes.byref(r)), "spread_task_reduce")
        self._results.append(r)
        return r

    def exit(self, a, B) -> None:
        """target exit data spread map(from: A[start:size]) depend(in: A[start:size]) nowait, into B."""
        import numpy as np

        if not (isinstance(B, np.ndarray) and B.dtype == np.float64 and B.flags["C_CONTIGUOUS"]):
            raise TypeError("exit: B must be a C-contiguous float64 array")
        self._keep.append(B)
        N.check(N.lib().spread_exit_data(self._h, a, B.ctypes.data_as(ctypes.POINTER(ctypes.c_double))),
                "spread_exit_data")

    def taskwait(self) -> None:
        N.check(N.lib().spread_taskwait(self._h), "spread_taskwait")
        self._keep = []

    def hold(self, chunk: int) -> None:
        """Test hook: chunk's stream waits before its next task until release()."""
        N.check(N.lib().spread_tasks_hold(self._h, int(chunk)), "spread_tasks_hold")

    def release(self) -> None:
        N.check(N.lib().spread_tasks_release(self._h), "spread_tasks_release")

    def set_trace(self, on: bool = True) -> None:
        N.check(N.lib().spread_tasks_set_trace(self._h, 1 if on else 0), "spread_tasks_set_trace")

    def trace(self) -> list:
        """[(chunk, kind, start_ms, end_ms)] of every traced chunk task (waits first)."""
        cnt = ctypes.c_int64()
        N.check(N.lib().spread_tasks_trace(self._h, None, 0, ctypes.byref(cnt)), "spread_tasks_trace")
        recs = (N.spread_task_record * max(1, cnt.value))()
        N.check(N.lib().spread_tasks_trace(self._h, recs, cnt.value, ctypes.byref(cnt)), "spread_tasks_trace")
        return [(r.chunk, self.KINDS[r.kind], r.start_ms, r.end_ms) for r in recs[:cnt.value]]

