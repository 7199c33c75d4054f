"""Exact-stats domain (S18; include/somier.h, somier_stats): the
kernels' centre sums are exact while every position is finite with
|x| < 2^23 (C + h stays in [2^52, 2^53), stats.cuh). Each state carries an
upper bound on max |x| (stats_layout.hpp, xbound_step): exact for a state the
stats kernels sum (init / load) or the host-streamed mode maps in, and
(B + sqrt(vmax2) |dt|) (1 + 2^-40) for the state a step produces. A state
whose bound reaches 2^23 reports a NaN centre instead of possibly wrong
finite sums. The oracle's sums are the exact definition at any finite x
(int128 of nearbyint(x 2^60)), so inside the domain the GPU's stats must equal
them bit for bit; the bound chain is recomputed here from the oracle's states
and vmax (bitwise the GPU's), with a 1e-12 band for the device's contracted
arithmetic."""
import math
import struct

import numpy as np
import pytest

import oracle as O

pytestmark = pytest.mark.gpu
P = pytest.importorskip("paper_conf_ipps_torresft22_b200")
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _op(sp):
    return O.Params(n=sp.n, spacing=sp.spacing, rest_len=sp.rest_len, k_spring=sp.k_spring, mass=sp.mass,
                    dt=sp.dt, amplitude=sp.amplitude, seed=sp.seed)


def _xmax(s):
    X = np.abs(np.stack([s.x, s.y, s.z]))
    return math.nan if np.isnan(X).any() else float(X.max())


def _bounds(x0max, stats, dt):
    """Bound of state 0 (exact max |x|) and of each state after it."""
    out = [x0max]
    for st in stats:
        v2 = struct.unpack("<d", struct.pack("<Q", st.vmax2_bits))[0]
        out.append((out[-1] + math.sqrt(v2) * abs(dt)) * (1.0 + 2.0 ** -40))
    return out


def _check(st, ref_stats, bound):
    assert st.vmax2_bits == ref_stats.vmax2_bits or (math.isnan(st.vmax) and math.isnan(ref_stats.vmax))
    if not bound < 2.0 ** 23 * (1 + 1e-12):  # NaN included
        assert not st.in_domain and all(math.isnan(c) for c in st.centre)
    elif bound < 2.0 ** 23 * (1 - 1e-12):
        assert st.in_domain
        assert st.sums == ref_stats.sums and st.centre == ref_stats.centre


@pytest.mark.parametrize("kernel", [P.K1_TB2, P.K1_MARCH2, P.K1_MARCH, P.K1_DIRECT])
@pytest.mark.parametrize("xbig", [2.0 ** 23 - 1.0, -(2.0 ** 23), 2.0 ** 23, -(2.0 ** 23) - 1.0, 3e30, math.inf])
def test_loaded_state_and_next_steps(kernel, xbig):
    """One interior node's x set to xbig by somier_load (stats of the loaded
    state: the stats kernel), then two steps (K1: both of K1_TB2's steps)."""
    n = (10, 11, 34)
    sp = P.SomierParams(n=n, seed=3, kernel=kernel)
    s0 = O.init(_op(sp))
    s0.x[4, 5, 17] = xbig
    ref = [(s0, O.centers(s0))]
    for _ in range(2):
        ref.append(O.step(ref[-1][0]))
    X = np.stack([s0.x, s0.y, s0.z])
    V = np.stack([s0.vx, s0.vy, s0.vz])
    with P.Somier(P.Spread([0], 1, n[0] - 2), sp) as s:
        assert s.kernel_in_use == kernel
        s.load(X, V)
        _check(s.stats(), ref[0][1], _xmax(s0))
        s.step(2)
        hist = s.stats_history(0, 3)
        Xg, Vg = s.read()
    b = _bounds(_xmax(s0), [r[1] for r in ref[1:]], sp.dt)
    for t in range(3):
        _check(hist[t], ref[t][1], b[t])
    with np.errstate(invalid="ignore"):
        same = (Xg == np.stack([ref[2][0].x, ref[2][0].y, ref[2][0].z])) | (np.isnan(Xg) & np.isnan(
            np.stack([ref[2][0].x, ref[2][0].y, ref[2][0].z])))
    assert same.all()


@pytest.mark.parametrize("kernel", [P.K1_TB2, P.K1_MARCH2])
def test_diverging_run(kernel):
    """An unstable time step (dt far beyond 2/omega): the amplitude grows by
    orders of magnitude per step and leaves the domain; every step's stats are
    exact while the state is inside it and NaN once a node is outside."""
    n = (12, 13, 40)
    sp = P.SomierParams(n=n, seed=4, dt=0.9, kernel=kernel)
    ref = [(O.init(_op(sp)), None)]
    ref[0] = (ref[0][0], O.centers(ref[0][0]))
    for _ in range(12):
        ref.append(O.step(ref[-1][0]))
    b = _bounds(_xmax(ref[0][0]), [r[1] for r in ref[1:]], sp.dt)
    assert b[0] < 2.0 ** 23 and b[3] < 2.0 ** 23 and not b[-1] < 2.0 ** 23, "must start inside and leave"
    with P.Somier(P.Spread([0], 1, n[0] - 2), sp) as s:
        s.step(12)
        hist = s.stats_history(0, 13)
    for t in range(13):
        _check(hist[t], ref[t][1], b[t])


def test_stream_mode_diverging():
    """The host-streamed Somier sums its states with the same kernels: NaN
    centres once the state leaves the domain, exact stats before."""
    n = (12, 13, 40)
    sp = P.SomierParams(n=n, seed=4, dt=0.9)
    ref = [O.init(_op(sp))]
    stats = []
    for _ in range(12):
        s, st = O.step(ref[-1])
        ref.append(s)
        stats.append(st)
    spread = P.Spread([0], 1, n[0] - 2, chunk=3)
    with P.SomierStream(spread, sp, buffers=2) as ss:
        X, V = ss.generate()
        XN = np.zeros_like(X)
        got = ss.run(X, V, XN, 12)
    b = _bounds(_xmax(ref[0]), stats, sp.dt)
    assert b[3] < 2.0 ** 23 and not b[-1] < 2.0 ** 23
    for t in range(12):
        _check(got[t], stats[t], b[t + 1])
