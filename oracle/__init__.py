"""CPU oracle for the Somier time step -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference legs may import this package. The product package
(paper_conf_ipps_torresft22_b200) never imports it; the two share no code.

Thin ctypes marshalling over oracle/liboracle.so (somier_oracle.c), which is
the plain sequential fp64 implementation of PAPER.md §V (lines 319-344): the
forces -> accelerations -> velocities -> positions -> centers kernels
 with the readings listed in DESIGN.md §3.
"""
from __future__ import annotations

import ctypes
import dataclasses
import os

import numpy as np

from . import build_oracle

_lib = None


class _Params(ctypes.Structure):
    _fields_ = [
        ("n", ctypes.c_int64 * 3),
        ("spacing", ctypes.c_double),
        ("rest_len", ctypes.c_double),
        ("k_spring", ctypes.c_double),
        ("mass", ctypes.c_double),
        ("dt", ctypes.c_double),
        ("amplitude", ctypes.c_double),
        ("seed", ctypes.c_uint64),
    ]


class _Stats(ctypes.Structure):
    _fields_ = [
        ("centre", ctypes.c_double * 3),
        ("vmax", ctypes.c_double),
        ("sum_lo", ctypes.c_uint64 * 3),
        ("sum_hi", ctypes.c_int64 * 3),
        ("vmax2_bits", ctypes.c_uint64),
    ]


@dataclasses.dataclass
class Params:
    """Somier parameters; defaults are SURVEY §8(c) item 7 (reading S3)."""

    n: tuple = (16, 16, 16)
    spacing: float = 1.0
    rest_len: float = 1.0
    k_spring: float = 10.0
    mass: float = 1.0
    dt: float = 1e-3
    amplitude: float = 0.05
    seed: int = 1

    def c(self) -> _Params:
        p = _Params()
        for d in range(3):
            p.n[d] = int(self.n[d])
        p.spacing, p.rest_len, p.k_spring = self.spacing, self.rest_len, self.k_spring
        p.mass, p.dt, p.amplitude, p.seed = self.mass, self.dt, self.amplitude, int(self.seed)
        return p


@dataclasses.dataclass
class Stats:
    centre: tuple
    vmax: float
    sums: tuple  # exact int128 fixed-point sums (units of 2^-60)
    vmax2_bits: int


def lib():
    global _lib
    if _lib is None:
        # ORACLE_LIB: an alternative build of somier_oracle.c (tools/mutate_oracle.py
        # points it at deliberately broken mutants to show the pins catch them)
        _lib = _bind(ctypes.CDLL(os.environ.get("ORACLE_LIB") or build_oracle.build()))
    return _lib


_lib_omp = None


def lib_omp():
    """The optional all-cores build of the same source (-fopenmp): bench.py's
    second CPU-baseline line. OMP_NUM_THREADS applies when it is first loaded."""
    global _lib_omp
    if _lib_omp is None:
        _lib_omp = _bind(ctypes.CDLL(build_oracle.build_omp()))
    return _lib_omp


def _bind(L):
    dp = ctypes.POINTER(ctypes.c_double)
    P = ctypes.POINTER(_Params)
    S = ctypes.POINTER(_Stats)
    L.oracle_splitmix64_at.restype = ctypes.c_uint64
    L.oracle_splitmix64_at.argtypes = [ctypes.c_uint64, ctypes.c_uint64]
    L.oracle_rest_position.argtypes = [P, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, dp]
    L.oracle_init.argtypes = [P] + [dp] * 6
    i64a = ctypes.POINTER(ctypes.c_int64)
    L.oracle_init_window.argtypes = [P, i64a, i64a] + [dp] * 6
    L.oracle_spring.argtypes = [dp, dp, ctypes.c_double, ctypes.c_double, dp]
    for name in ("oracle_acceleration_1", "oracle_velocity_1", "oracle_position_1"):
        fn = getattr(L, name)
        fn.restype = ctypes.c_double
    L.oracle_acceleration_1.argtypes = [ctypes.c_double, ctypes.c_double]
    L.oracle_velocity_1.argtypes = [ctypes.c_double] * 3
    L.oracle_position_1.argtypes = [ctypes.c_double] * 3
    L.oracle_forces.argtypes = [P] + [dp] * 6
    L.oracle_accelerations.argtypes = [P] + [dp] * 6
    L.oracle_velocities.argtypes = [P] + [dp] * 6
    L.oracle_positions.argtypes = [P] + [dp] * 9
    L.oracle_centers.argtypes = [P] + [dp] * 6 + [S]
    L.oracle_step.argtypes = [P] + [dp] * 9 + [S]
    L.oracle_run.argtypes = [P, ctypes.c_int64] + [dp] * 6 + [S]
    L.oracle_run_timed.argtypes = [P, ctypes.c_int64] + [dp] * 6 + [S, dp]
    L.oracle_threads.restype = ctypes.c_int
    L.oracle_stencil3.argtypes = [dp, dp, ctypes.c_int64]
    return L


def _ptr(a: np.ndarray):
    assert a.dtype == np.float64 and a.flags["C_CONTIGUOUS"]
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def _stats(s: _Stats) -> Stats:
    sums = []
    for c in range(3):
        sums.append((int(s.sum_hi[c]) << 64) | int(s.sum_lo[c]))
    return Stats(tuple(s.centre), float(s.vmax), tuple(sums), int(s.vmax2_bits))


class State:
    """Full-grid state: X = (x, y, z) and V = (vx, vy, vz), each an (n0,n1,n2) fp64 grid."""

    def __init__(self, p: Params, x, y, z, vx, vy, vz):
        self.p = p
        self.x, self.y, self.z, self.vx, self.vy, self.vz = x, y, z, vx, vy, vz

    @property
    def X(self):
        return np.stack([self.x, self.y, self.z])

    @property
    def V(self):
        return np.stack([self.vx, self.vy, self.vz])

    def copy(self) -> "State":
        return State(self.p, *(a.copy() for a in (self.x, self.y, self.z, self.vx, self.vy, self.vz)))


def splitmix64_at(seed: int, idx: int) -> int:
    return int(lib().oracle_splitmix64_at(seed, idx))


def rest_position(p: Params, i: int, j: int, k: int):
    out = (ctypes.c_double * 3)()
    lib().oracle_rest_position(ctypes.byref(p.c()), i, j, k, out)
    return tuple(out)


def empty(p: Params) -> State:
    shape = tuple(int(v) for v in p.n)
    return State(p, *(np.zeros(shape, np.float64) for _ in range(6)))


def init(p: Params) -> State:
    s = empty(p)
    rc = lib().oracle_init(ctypes.byref(p.c()), *(_ptr(a) for a in (s.x, s.y, s.z, s.vx, s.vy, s.vz)))
    if rc != 0:
        raise ValueError("oracle_init rejected parameters %r" % (p,))
    return s


def init_window(p: Params, lo, w) -> State:
    """Initial state of the global grid p.n restricted to [lo, lo+w); the returned
    State is a standalone grid of shape w (its Params carry n = w)."""
    sub = Params(n=tuple(int(v) for v in w), spacing=p.spacing, rest_len=p.rest_len, k_spring=p.k_spring,
                 mass=p.mass, dt=p.dt, amplitude=p.amplitude, seed=p.seed)
    s = empty(sub)
    lo_a = (ctypes.c_int64 * 3)(*[int(v) for v in lo])
    w_a = (ctypes.c_int64 * 3)(*[int(v) for v in w])
    rc = lib().oracle_init_window(ctypes.byref(p.c()), lo_a, w_a,
                                  *(_ptr(a) for a in (s.x, s.y, s.z, s.vx, s.vy, s.vz)))
    if rc != 0:
        raise ValueError("oracle_init_window rejected the window")
    return s


def spring(xp, xq, K: float, L: float):
    a = (ctypes.c_double * 3)(*xp)
    b = (ctypes.c_double * 3)(*xq)
    g = (ctypes.c_double * 3)()
    lib().oracle_spring(a, b, K, L, g)
    return tuple(g)


def acceleration_1(f: float, m: float) -> float:
    return lib().oracle_acceleration_1(f, m)


def velocity_1(v: float, a: float, dt: float) -> float:
    return lib().oracle_velocity_1(v, a, dt)


def position_1(x: float, v: float, dt: float) -> float:
    return lib().oracle_position_1(x, v, dt)


def forces(s: State):
    f = [np.zeros_like(s.x) for _ in range(3)]
    lib().oracle_forces(ctypes.byref(s.p.c()), _ptr(s.x), _ptr(s.y), _ptr(s.z), *(_ptr(a) for a in f))
    return f


def accelerations(p: Params, f):
    a = [np.zeros_like(f[0]) for _ in range(3)]
    lib().oracle_accelerations(ctypes.byref(p.c()), *(_ptr(v) for v in f), *(_ptr(v) for v in a))
    return a


def velocities(p: Params, a, v):
    lib().oracle_velocities(ctypes.byref(p.c()), *(_ptr(t) for t in a), *(_ptr(t) for t in v))


def positions(p: Params, x, v):
    xn = [np.zeros_like(x[0]) for _ in range(3)]
    lib().oracle_positions(ctypes.byref(p.c()), *(_ptr(t) for t in x), *(_ptr(t) for t in v),
                           *(_ptr(t) for t in xn))
    return xn


def centers(s: State) -> Stats:
    st = _Stats()
    lib().oracle_centers(ctypes.byref(s.p.c()), *(_ptr(a) for a in (s.x, s.y, s.z, s.vx, s.vy, s.vz)),
                         ctypes.byref(st))
    return _stats(st)


def step(s: State) -> tuple:
    """One time step; returns (new State, Stats). The input state is not modified."""
    out = s.copy()
    xn = [np.zeros_like(s.x) for _ in range(3)]
    st = _Stats()
    rc = lib().oracle_step(ctypes.byref(s.p.c()), _ptr(s.x), _ptr(s.y), _ptr(s.z),
                           _ptr(out.vx), _ptr(out.vy), _ptr(out.vz), *(_ptr(a) for a in xn),
                           ctypes.byref(st))
    if rc != 0:
        raise ValueError("oracle_step failed")
    out.x, out.y, out.z = xn
    return out, _stats(st)


def run_timed(s: State, nsteps: int, omp: bool = False) -> tuple:
    """nsteps steps on a copy of s with the C step loop timed by the steady clock
    (oracle_run_timed); returns (final State, Stats of the last step, seconds,
    threads). omp: the all-cores build of the same source."""
    L = lib_omp() if omp else lib()
    out = s.copy()
    st = _Stats()
    sec = ctypes.c_double()
    rc = L.oracle_run_timed(ctypes.byref(s.p.c()), int(nsteps),
                            *(_ptr(a) for a in (out.x, out.y, out.z, out.vx, out.vy, out.vz)),
                            ctypes.byref(st), ctypes.byref(sec))
    if rc != 0:
        raise ValueError("oracle_run_timed failed")
    return out, _stats(st), sec.value, int(L.oracle_threads())


def run(s: State, nsteps: int) -> tuple:
    """nsteps steps on a copy of s; returns (final State, Stats of the last step)."""
    out = s.copy()
    st = _Stats()
    rc = lib().oracle_run(ctypes.byref(s.p.c()), int(nsteps),
                          *(_ptr(a) for a in (out.x, out.y, out.z, out.vx, out.vy, out.vz)),
                          ctypes.byref(st))
    if rc != 0:
        raise ValueError("oracle_run failed")
    return out, _stats(st)


def stencil3(a: np.ndarray) -> np.ndarray:
    a = np.ascontiguousarray(a, dtype=np.float64)
    b = np.zeros_like(a)
    lib().oracle_stencil3(_ptr(a), _ptr(b), a.size)
    return b


def reduce_exact(a, start: int, length: int, op: str = "sum", scale_exp: int = 60):
    """The reduction clause's result by definition (S15 generalised;
    PAPER.md:330, 773): "sum" -> (value, S) with S = sum over i in
    [start, start+length) of round_half_even(a[i] * 2^scale_exp), computed with
    Python integers and Fractions (exact), value = S * 2^-scale_exp rounded once;
    "min" / "max" -> (element, None) in the IEEE total order of non-NaN values
    (-0 < +0), NaN if any element is NaN; empty: 0 / +inf / -inf."""
    import math
    from fractions import Fraction

    xs = [float(v) for v in a[start:start + length]]
    if op == "sum":
        S = 0
        for x in xs:
            if not math.isfinite(x) or abs(Fraction(x) * Fraction(2) ** scale_exp) >= 2 ** 94:
                raise ValueError("outside the exact domain")
            S += round(Fraction(x) * Fraction(2) ** scale_exp)  # Python rounds half to even
        return float(Fraction(S) / Fraction(2) ** scale_exp), S
    if any(math.isnan(x) for x in xs):
        return math.nan, None
    if not xs:
        return (math.inf if op == "min" else -math.inf), None
    key = lambda x: (x, math.copysign(1.0, x))  # noqa: E731  -0 before +0
    return (min(xs, key=key) if op == "min" else max(xs, key=key)), None


def lib_path() -> str:
    return os.path.join(os.path.dirname(os.path.abspath(__file__)), "liboracle.so")
