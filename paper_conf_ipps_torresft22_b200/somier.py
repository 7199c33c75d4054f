"""The Somier time step spread over devices (include/somier.h; §V).

A thin ctypes layer: parameters in, pointers and sizes across the C ABI, and
numpy views out. The step itself runs in libsomier.so's sm_100a kernels.
"""
from __future__ import annotations

import ctypes
import dataclasses
from typing import Optional, Sequence, Tuple

import numpy as np

from . import _native as N
from .spread import Spread


@dataclasses.dataclass
class SomierParams:
    """Defaults are DESIGN.md §3 reading S3."""

    n: Tuple[int, int, int] = (16, 16, 16)
    spacing: float = 1.0
    rest_len: float = 1.0
    k_spring: float = 10.0
    mass: float = 1.0
    dt: float = 1e-3
    amplitude: float = 0.05
    seed: int = 42
    kernel: int = N.K1_AUTO
    exchange: int = 0  # somier_exchange: FUSED (0), COPY (1), NCCL (2)
    math: int = 0  # somier_math: EXACT (0, bit-identical to the oracle) or FMA (1, reading S22)

    def c(self) -> N.somier_params:
        p = N.somier_params()
        for d in range(3):
            p.n[d] = int(self.n[d])
        p.spacing, p.rest_len, p.k_spring, p.mass = self.spacing, self.rest_len, self.k_spring, self.mass
        p.dt, p.amplitude, p.seed, p.kernel = self.dt, self.amplitude, int(self.seed), int(self.kernel)
        p.exchange, p.math = int(self.exchange), int(self.math)
        return p

    @property
    def interior_nodes(self) -> int:
        return (self.n[0] - 2) * (self.n[1] - 2) * (self.n[2] - 2)


@dataclasses.dataclass
class Stats:
    step: int
    centre: Tuple[float, float, float]
    vmax: float
    sums: Tuple[int, int, int]    # exact int128 fixed-point sums, units of 2^-60
    vmax2_bits: int
    nodes: int

    @property
    def in_domain(self) -> bool:
        """False when a node of the state lies outside the exact-stats domain
        (|x| >= 2^23 or non-finite): the centre is then NaN (somier.h)."""
        return not any(c != c for c in self.centre)

    @staticmethod
    def from_c(s: N.somier_stats_t) -> "Stats":
        sums = tuple((int(s.sum_hi[c]) << 64) | int(s.sum_lo[c]) for c in range(3))
        return Stats(int(s.step), tuple(s.centre), float(s.vmax), sums, int(s.vmax2_bits), int(s.nodes))

    def to_c(self) -> N.somier_stats_t:
        s = N.somier_stats_t()
        s.step = self.step
        for c in range(3):
            s.centre[c] = self.centre[c]
            v = self.sums[c] & ((1 << 128) - 1)
            s.sum_lo[c] = v & ((1 << 64) - 1)
            hi = v >> 64
            s.sum_hi[c] = hi - (1 << 64) if hi >= (1 << 63) else hi
        s.vmax = self.vmax
        s.vmax2_bits = self.vmax2_bits
        s.nodes = self.nodes
        return s


def _dptr(a, count: int) -> ctypes.POINTER(ctypes.c_double):
    """numpy float64 C-contiguous array of exactly `count` elements (the C side
    reads or writes that many doubles), or an integer address (e.g. a pinned
    torch tensor's data_ptr(); the caller guarantees its size)."""
    if a is None:
        return None
    if isinstance(a, int):
        return ctypes.cast(ctypes.c_void_p(a), ctypes.POINTER(ctypes.c_double))
    if not (isinstance(a, np.ndarray) and a.dtype == np.float64 and a.flags["C_CONTIGUOUS"]):
        raise TypeError("expected a C-contiguous float64 numpy array or an address")
    if a.size != count:
        raise ValueError("grid has %d elements, the C ABI needs %d" % (a.size, count))
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def combine_stats(parts: Sequence[Stats], params: SomierParams) -> Stats:
    """Exact combination of per-process partial stats (somier_stats_combine)."""
    arr = (N.somier_stats_t * len(parts))(*[p.to_c() for p in parts])
    out = N.somier_stats_t()
    pc = params.c()
    N.check(N.lib().somier_stats_combine(arr, len(parts), ctypes.byref(pc), ctypes.byref(out)),
            "somier_stats_combine")
    return Stats.from_c(out)


class Somier:
    """A Somier grid spread over the devices of `spread`.

    device_pos=None: single-process mode (all chunks, all devices of the list).
    device_pos=q: multi-process mode, this process owns the chunks at list
    position q; call ipc_connect() with every process's ipc_export() blob.
    """

    def __init__(self, spread: Spread, params: SomierParams, device_pos: Optional[int] = None,
                 cuda_device: int = -1, cuda_devices: Optional[Sequence[int]] = None):
        L = N.lib()
        self.params = params
        self._cells = int(params.n[0]) * int(params.n[1]) * int(params.n[2])  # doubles per host grid
        self.spread = spread
        self._pc = params.c()
        h = ctypes.c_void_p()
        if cuda_devices is not None:
            arr = (ctypes.c_int * len(cuda_devices))(*cuda_devices)
            N.check(L.somier_init_on(spread.handle, ctypes.byref(self._pc), arr, ctypes.byref(h)), "somier_init_on")
        elif device_pos is None:
            N.check(L.somier_init(spread.handle, ctypes.byref(self._pc), ctypes.byref(h)), "somier_init")
        else:
            N.check(L.somier_init_local(spread.handle, ctypes.byref(self._pc), int(device_pos), int(cuda_device),
                                        ctypes.byref(h)), "somier_init_local")
        self._h = h
        self.device_pos = device_pos

    # -- lifetime ------------------------------------------------------------
    def close(self) -> None:
        if getattr(self, "_h", None):
            N.lib().somier_destroy(self._h)
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

    def _grids(self, grids):
        return [_dptr(g, self._cells) for g in grids]

    # -- the step ------------------------------------------------------------
    def step(self, nsteps: int = 1) -> None:
        N.check(N.lib().somier_step(self._h, int(nsteps)), "somier_step")

    def sync(self) -> None:
        N.check(N.lib().somier_sync(self._h), "somier_sync")

    def stats(self) -> Stats:
        out = N.somier_stats_t()
        N.check(N.lib().somier_stats(self._h, ctypes.byref(out)), "somier_stats")
        return Stats.from_c(out)

    def stats_history(self, first_step: int, count: int) -> list:
        """Stats after steps first_step .. first_step+count-1 (somier_stats_history):
        every step's centres / vmax, from the device-side history ring."""
        count = int(count)
        out = (N.somier_stats_t * max(1, count))()
        N.check(N.lib().somier_stats_history(self._h, int(first_step), count, out), "somier_stats_history")
        return [Stats.from_c(out[i]) for i in range(count)]

    def set_timing(self, on: bool = True) -> None:
        """somier_set_timing: bracket every launch with events (waits / kernel)."""
        N.check(N.lib().somier_set_timing(self._h, 1 if on else 0), "somier_set_timing")

    def take_timing(self) -> dict:
        """somier_take_timing: launches, summed and largest flag-wait and kernel ms since the last take."""
        t = N.somier_timing_t()
        N.check(N.lib().somier_take_timing(self._h, ctypes.byref(t)), "somier_take_timing")
        return {"launches": t.launches, "wait_ms": t.wait_ms, "kernel_ms": t.kernel_ms,
                "wait_max_ms": t.wait_max_ms, "kernel_max_ms": t.kernel_max_ms}

    # -- data movement -------------------------------------------------------
    def read(self, X=None, V=None):
        """Copy the owned planes into host grids; returns (X, V), each (3, n0, n1, n2)."""
        shape = (3,) + tuple(int(v) for v in self.params.n)
        if X is None:
            X = np.zeros(shape, np.float64)
        if V is None:
            V = np.zeros(shape, np.float64)
        ptrs = [_dptr(X[c], self._cells) for c in range(3)] + [_dptr(V[c], self._cells) for c in range(3)]
        N.check(N.lib().somier_read(self._h, *ptrs), "somier_read")
        return X, V

    def read_planes(self, i0: int, count: int, X=None, V=None):
        """target update spread from(X[i0:count], V[i0:count]): returns (X, V), each (3, count, n1, n2)."""
        shape = (3, int(count), int(self.params.n[1]), int(self.params.n[2]))
        X = np.zeros(shape, np.float64) if X is None else X
        V = np.zeros(shape, np.float64) if V is None else V
        m = int(count) * int(self.params.n[1]) * int(self.params.n[2])
        ptrs = [_dptr(X[c], m) for c in range(3)] + [_dptr(V[c], m) for c in range(3)]
        N.check(N.lib().somier_read_planes(self._h, int(i0), int(count), *ptrs), "somier_read_planes")
        return X, V

    def read_ptrs(self, ptrs: Sequence[int]) -> None:
        N.check(N.lib().somier_read(self._h, *self._grids(ptrs)), "somier_read")

    def load(self, X, V) -> None:
        ptrs = ([_dptr(np.ascontiguousarray(X[c]), self._cells) for c in range(3)]
                + [_dptr(np.ascontiguousarray(V[c]), self._cells) for c in range(3)])
        self._keep = (X, V)
        N.check(N.lib().somier_load(self._h, *ptrs), "somier_load")

    def load_ptrs(self, ptrs: Sequence[int]) -> None:
        N.check(N.lib().somier_load(self._h, *self._grids(ptrs)), "somier_load")

    # -- multi-process -------------------------------------------------------
    def ipc_export(self) -> bytes:
        n = ctypes.c_size_t()
        N.check(N.lib().somier_ipc_export(self._h, None, 0, ctypes.byref(n)), "somier_ipc_export")
        buf = ctypes.create_string_buffer(n.value)
        N.check(N.lib().somier_ipc_export(self._h, buf, n.value, ctypes.byref(n)), "somier_ipc_export")
        return buf.raw[: n.value]

    def ipc_connect(self, blobs: Sequence[bytes]) -> None:
        bufs = [ctypes.create_string_buffer(b, len(b)) for b in blobs]
        ptrs = (ctypes.c_void_p * len(bufs))(*[ctypes.cast(b, ctypes.c_void_p) for b in bufs])
        lens = (ctypes.c_size_t * len(bufs))(*[len(b) for b in blobs])
        N.check(N.lib().somier_ipc_connect(self._h, ptrs, lens, len(bufs)), "somier_ipc_connect")

    # -- streams / counters --------------------------------------------------
    def set_stream(self, device_pos: int, stream_ptr: int) -> None:
        N.check(N.lib().somier_set_stream(self._h, device_pos, ctypes.c_void_p(stream_ptr)), "somier_set_stream")

    def get_stream(self, device_pos: int) -> int:
        v = ctypes.c_void_p()
        N.check(N.lib().somier_get_stream(self._h, device_pos, ctypes.byref(v)), "somier_get_stream")
        return v.value or 0

    def _i64(self, fn, name) -> int:
        v = ctypes.c_int64()
        N.check(fn(self._h, ctypes.byref(v)), name)
        return v.value

    @property
    def step_count(self) -> int:
        return self._i64(N.lib().somier_step_count, "somier_step_count")

    @property
    def local_chunks(self) -> int:
        return self._i64(N.lib().somier_local_chunks, "somier_local_chunks")

    @property
    def launches(self) -> int:
        return self._i64(N.lib().somier_launch_count, "somier_launch_count")

    @property
    def device_bytes(self) -> int:
        return self._i64(N.lib().somier_device_bytes, "somier_device_bytes")

    @property
    def kernel_in_use(self) -> int:
        """The K1 implementation multi-step calls run (K1_TB2 / K1_MARCH2 / ...)."""
        v = ctypes.c_int32()
        N.check(N.lib().somier_kernel_in_use(self._h, ctypes.byref(v)), "somier_kernel_in_use")
        return v.value


class SomierStream:
    """Host-streamed Somier (include/somier.h, somier_stream_*): the state lives
    in host memory and each step maps every chunk of `spread` to its device,
    runs the fused step and maps the result back -- the paper's experiment
    (§V-A..C). buffers=1: One Buffer; >= 2: double buffering."""

    def __init__(self, spread: Spread, params: SomierParams, buffers: int = 2,
                 cuda_devices: Optional[Sequence[int]] = None):
        self.params = params
        self._cells = int(params.n[0]) * int(params.n[1]) * int(params.n[2])  # doubles per host grid
        self.spread = spread
        self._pc = params.c()
        h = ctypes.c_void_p()
        arr = None if cuda_devices is None else (ctypes.c_int * len(cuda_devices))(*cuda_devices)
        N.check(N.lib().somier_stream_create_on(spread.handle, ctypes.byref(self._pc), int(buffers), arr,
                                                ctypes.byref(h)), "somier_stream_create")
        self._h = h

    def close(self) -> None:
        if getattr(self, "_h", None):
            N.lib().somier_stream_destroy(self._h)
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

    def _grids(self, grids):
        return [_dptr(g, self._cells) for g in grids]

    def generate(self, X=None, V=None):
        """Initial state (bit-identical to Somier's) into host grids; returns (X, V)."""
        shape = (3,) + tuple(int(v) for v in self.params.n)
        X = np.zeros(shape, np.float64) if X is None else X
        V = np.zeros(shape, np.float64) if V is None else V
        self.generate_ptrs([X[0], X[1], X[2], V[0], V[1], V[2]])
        return X, V

    def generate_ptrs(self, grids) -> None:
        N.check(N.lib().somier_stream_generate(self._h, *self._grids(grids)), "somier_stream_generate")

    def step(self, X, V, XN) -> Stats:
        """One step: X (3 grids, read), V (3 grids, updated in place), XN (3 grids, written)."""
        return self.step_ptrs([X[0], X[1], X[2]], [V[0], V[1], V[2]], [XN[0], XN[1], XN[2]])

    def step_ptrs(self, X, V, XN) -> Stats:
        out = N.somier_stats_t()
        N.check(N.lib().somier_stream_step(self._h, *self._grids(X), *self._grids(V),
                                           *self._grids(XN), ctypes.byref(out)), "somier_stream_step")
        return Stats.from_c(out)

    def run(self, X, V, XN, nsteps: int, stats: bool = True):
        """nsteps steps with chunk-level dependencies (somier_stream_run): X and
        XN are used alternately, X_{nsteps} ends in X if nsteps is even, else in
        XN. Returns the per-step Stats (or None)."""
        return self.run_ptrs([X[0], X[1], X[2]], [V[0], V[1], V[2]], [XN[0], XN[1], XN[2]], nsteps, stats)

    def run_ptrs(self, X, V, XN, nsteps: int, stats: bool = True):
        out = (N.somier_stats_t * max(1, int(nsteps)))() if stats else None
        N.check(N.lib().somier_stream_run(self._h, *self._grids(X), *self._grids(V),
                                          *self._grids(XN), int(nsteps), out), "somier_stream_run")
        return [Stats.from_c(out[t]) for t in range(int(nsteps))] if stats else None

    def traffic(self):
        a, b, c = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
        N.check(N.lib().somier_stream_traffic(self._h, ctypes.byref(a), ctypes.byref(b), ctypes.byref(c)),
                "somier_stream_traffic")
        return {"h2d_bytes": a.value, "d2h_bytes": b.value, "launches": c.value}

    def run2(self, X, V, XN, VN, nsteps: int, stats: bool = True):
        """nsteps steps, two per host round trip (somier_stream_run2): (X, V) and
        (XN, VN) are used alternately per launch; the final state is in (X, V)
        if the number of launches ceil(nsteps / 2) is even, else in (XN, VN).
        Returns the Stats after each step (or None)."""
        return self.run2_ptrs([X[0], X[1], X[2]], [V[0], V[1], V[2]], [XN[0], XN[1], XN[2]],
                              [VN[0], VN[1], VN[2]], nsteps, stats)

    def run2_ptrs(self, X, V, XN, VN, nsteps: int, stats: bool = True):
        out = (N.somier_stats_t * max(1, int(nsteps)))() if stats else None
        N.check(N.lib().somier_stream_run2(self._h, *self._grids(X), *self._grids(V),
                                           *self._grids(XN), *self._grids(VN), int(nsteps), out),
                "somier_stream_run2")
        return [Stats.from_c(out[t]) for t in range(int(nsteps))] if stats else None

    def traffic2(self):
        """Host<->device bytes of one two-step launch of run2."""
        a, b = ctypes.c_int64(), ctypes.c_int64()
        N.check(N.lib().somier_stream_traffic2(self._h, ctypes.byref(a), ctypes.byref(b)), "somier_stream_traffic2")
        return {"h2d_bytes": a.value, "d2h_bytes": b.value}

    def run_blocked(self, X, V, XN, VN, nsteps: int, steps_per_trip: int, stats: bool = True):
        """nsteps steps, `steps_per_trip` per host round trip
        (somier_stream_run_blocked); buffers alternate per trip as in run2.
        Returns the Stats after each step (or None)."""
        return self.run_blocked_ptrs([X[0], X[1], X[2]], [V[0], V[1], V[2]], [XN[0], XN[1], XN[2]],
                                     [VN[0], VN[1], VN[2]], nsteps, steps_per_trip, stats)

    def run_blocked_ptrs(self, X, V, XN, VN, nsteps: int, steps_per_trip: int, stats: bool = True):
        s = int(steps_per_trip)
        out = (N.somier_stats_t * max(1, int(nsteps)))() if stats else None
        N.check(N.lib().somier_stream_run_blocked(self._h, *self._grids(X), *self._grids(V),
                                                  *self._grids(XN), *self._grids(VN), int(nsteps), s,
                                                  out), "somier_stream_run_blocked")
        return [Stats.from_c(out[t]) for t in range(int(nsteps))] if stats else None

    def chunk_counts(self) -> list:
        """Chunk tasks each list position has run (somier_stream_chunk_counts)."""
        n = len(self.spread.devices)
        arr = (ctypes.c_int64 * n)()
        N.check(N.lib().somier_stream_chunk_counts(self._h, arr), "somier_stream_chunk_counts")
        return list(arr)

    def set_delay(self, device_pos: int, ns: int) -> None:
        """Test hook: position device_pos spins >= ns per chunk task (somier_stream_set_delay)."""
        N.check(N.lib().somier_stream_set_delay(self._h, int(device_pos), int(ns)), "somier_stream_set_delay")

    def traffic_blocked(self, steps_per_trip: int):
        """Host<->device bytes of one trip of run_blocked with steps_per_trip steps."""
        a, b = ctypes.c_int64(), ctypes.c_int64()
        N.check(N.lib().somier_stream_traffic_blocked(self._h, int(steps_per_trip), ctypes.byref(a), ctypes.byref(b)),
                "somier_stream_traffic_blocked")
        return {"h2d_bytes": a.value, "d2h_bytes": b.value}
