"""SOMIER_MATH_FMA (include/somier.h, reading S22): the contraction
north_star allows -- "max relative error <= 1e-10 on positions and velocities
after 100 steps (fp64, FMA contraction the only allowed difference).
Partitioned runs must be bit-identical to the 1-GPU run."

The uncontracted oracle stays the reference. In FMA mode the GPU state is held
to the 1e-10 bar against it (normwise, and on the displacement X - X0, reading
S12), must actually differ from it (the mode is live), and must be
bit-identical across kernels, chunkings, logical device lists and the
host-streamed mode. The stats keep their exact definition: they are checked
bitwise against the oracle's `centers` applied to the GPU's own FMA state."""
import numpy as np
import pytest

import oracle as O

pytestmark = pytest.mark.gpu

P = pytest.importorskip("paper_conf_ipps_torresft22_b200")
torch = pytest.importorskip("torch")

KERNELS = [P.K1_DIRECT, P.K1_MARCH, P.K1_MARCH2, P.K1_TB2]


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _params(n, kernel=P.K1_AUTO, math=P.MATH_FMA, **kw):
    kw.setdefault("seed", 1)
    return P.SomierParams(n=tuple(n), kernel=kernel, math=math, **kw)


def _op(sp):
    return O.Params(n=sp.n, spacing=sp.spacing, rest_len=sp.rest_len, k_spring=sp.k_spring, mass=sp.mass,
                    dt=sp.dt, amplitude=sp.amplitude, seed=sp.seed)


def _run(sp, steps, devices=(0,), chunk=0, cuda_devices=None, history=False):
    spread = P.Spread(list(devices), 1, sp.n[0] - 2, chunk=chunk)
    kw = {} if cuda_devices is None else {"cuda_devices": cuda_devices}
    with P.Somier(spread, sp, **kw) as s:
        s.step(steps)
        st = s.stats()
        hist = s.stats_history(1, steps) if history else None
        X, V = s.read()
    return X, V, st, hist


def _rel(a, b):
    den = np.max(np.abs(b))
    return np.max(np.abs(a - b)) / den if den > 0 else np.max(np.abs(a - b))


def _state(sp, X, V):
    return O.State(_op(sp), X[0].copy(), X[1].copy(), X[2].copy(), V[0].copy(), V[1].copy(), V[2].copy())


_CACHE = {}


def _oracle(sp, steps):
    key = (sp.n, sp.seed, sp.mass, sp.spacing, sp.rest_len, sp.k_spring, sp.dt, sp.amplitude, steps)
    if key not in _CACHE:
        _CACHE[key] = O.run(O.init(_op(sp)), steps)
    return _CACHE[key]


def _within_bar(sp, X, V, steps):
    ref, _ = _oracle(sp, steps)
    x0 = O.init(_op(sp)).X
    ex, ed, ev = _rel(X, ref.X), _rel(X - x0, ref.X - x0), _rel(V, ref.V)
    assert ex <= 1e-10 and ed <= 1e-10 and ev <= 1e-10, (ex, ed, ev)
    return ref, (ex, ed, ev)


@pytest.mark.parametrize("kernel", KERNELS)
def test_fma_128cube_100_steps_within_bar(kernel):
    """configs[1] (128^3, 100 steps) in FMA mode: within 1e-10 of the oracle,
    yet not bit-identical to it (the contractions are live), and the stats are
    the exact definition applied to the FMA state."""
    sp = _params((128, 128, 128), kernel=kernel)
    X, V, st, _ = _run(sp, 100)
    ref, errs = _within_bar(sp, X, V, 100)
    assert not np.array_equal(X, ref.X) and not np.array_equal(V, ref.V), "FMA mode left the result unchanged"
    assert max(errs) > 0
    rst = O.centers(_state(sp, X, V))
    assert st.sums == rst.sums and st.vmax2_bits == rst.vmax2_bits and st.centre == rst.centre


@pytest.mark.parametrize("n", [(16, 16, 16), (17, 9, 33), (6, 131, 70), (4, 5, 260), (40, 33, 65)])
def test_fma_kernels_bit_identical(n):
    """Every K1 variant evaluates a node with the same contracted expressions."""
    out = []
    for kernel in KERNELS:
        sp = _params(n, kernel=kernel, seed=3)
        out.append(_run(sp, 11, history=True))
    X0, V0, st0, h0 = out[0]
    _within_bar(_params(n, seed=3), X0, V0, 11)
    for kernel, (X, V, st, h) in zip(KERNELS[1:], out[1:]):
        assert np.array_equal(X, X0) and np.array_equal(V, V0), kernel
        assert st.sums == st0.sums and st.vmax2_bits == st0.vmax2_bits, kernel
        assert [(a.sums, a.vmax2_bits) for a in h] == [(a.sums, a.vmax2_bits) for a in h0], kernel


@pytest.mark.parametrize("kernel", KERNELS)
def test_fma_non_unit_mass_and_spacing(kernel):
    """M != 1 (the division a = F/M stays exact), L != spacing (pre-stressed)."""
    kw = dict(mass=2.5, spacing=0.75, rest_len=0.8, k_spring=3.0, dt=2e-3, amplitude=0.1, seed=7)
    sp = _params((12, 14, 18), kernel=kernel, **kw)
    X, V, st, _ = _run(sp, 100)
    ref, _ = _within_bar(sp, X, V, 100)
    assert not np.array_equal(X, ref.X)
    ref_k = _run(_params((12, 14, 18), kernel=P.K1_DIRECT, **kw), 100)
    assert np.array_equal(X, ref_k[0]) and np.array_equal(V, ref_k[1])


@pytest.mark.parametrize("kernel", [P.K1_MARCH2, P.K1_TB2, P.K1_AUTO])
@pytest.mark.parametrize("layout", [dict(chunk=1), dict(chunk=3), dict(chunk=7),
                                    dict(devices=(0, 1), chunk=0, cuda_devices=[0, 0]),
                                    dict(devices=(2, 0, 1), chunk=5, cuda_devices=[0, 0, 0]),
                                    dict(devices=(0, 1, 2, 3), chunk=0, cuda_devices=[0, 0, 0, 0])])
def test_fma_partitions_bit_identical(kernel, layout):
    """Partitioned runs -- chunk tables on one device, logical device lists with
    the fused exchange between positions -- equal the one-chunk run bit for bit."""
    n, steps = (34, 21, 45), 9
    sp = _params(n, kernel=kernel, seed=11)
    X1, V1, st1, h1 = _run(sp, steps, history=True)
    X, V, st, h = _run(sp, steps, history=True, **layout)
    assert np.array_equal(X, X1) and np.array_equal(V, V1)
    assert [(a.sums, a.vmax2_bits) for a in h] == [(a.sums, a.vmax2_bits) for a in h1]


def test_fma_exchange_routes_bit_identical():
    n, steps = (26, 19, 37), 6
    base = _run(_params(n, kernel=P.K1_TB2, seed=5), steps)
    for ex in (P.EXCHANGE_FUSED, P.EXCHANGE_COPY):
        sp = _params(n, kernel=P.K1_TB2, seed=5, exchange=ex)
        X, V, _, _ = _run(sp, steps, devices=(0, 1, 2), chunk=0, cuda_devices=[0, 0, 0])
        assert np.array_equal(X, base[0]) and np.array_equal(V, base[1]), ex


def _pinned(shape):
    return torch.zeros(shape, dtype=torch.float64, pin_memory=True).numpy()


@pytest.mark.parametrize("mode", ["run", "run2", "blocked3"])
def test_fma_host_streamed_bit_identical(mode):
    """The host-streamed mode (somier_stream_*) with FMA equals the resident run."""
    n, nsteps = (20, 13, 37), 7
    sp = _params(n, seed=4)
    Xr, Vr, _, hr = _run(sp, nsteps, history=True)
    spread = P.Spread([0, 1], 1, n[0] - 2, chunk=3)
    with P.SomierStream(spread, sp, buffers=2, cuda_devices=[0, 0]) as s:
        X0, V0 = s.generate()
        X, V, XN, VN = _pinned(X0.shape), _pinned(V0.shape), _pinned(X0.shape), _pinned(V0.shape)
        X[...] = X0
        V[...] = V0
        if mode == "run":
            stats = s.run(X, V, XN, nsteps)
            fX, fV = (X, V) if nsteps % 2 == 0 else (XN, V)
        elif mode == "run2":
            stats = s.run2(X, V, XN, VN, nsteps)
            nl = nsteps // 2 + nsteps % 2
            fX, fV = (X, V) if nl % 2 == 0 else (XN, VN)
        else:
            stats = s.run_blocked(X, V, XN, VN, nsteps, 3)
            nt = -(-nsteps // 3)
            fX, fV = (X, V) if nt % 2 == 0 else (XN, VN)
    assert np.array_equal(fX, Xr) and np.array_equal(fV, Vr)
    assert [(a.sums, a.vmax2_bits) for a in stats] == [(a.sums, a.vmax2_bits) for a in hr]


def test_exact_mode_is_the_default_and_bitwise():
    sp = P.SomierParams(n=(16, 16, 16), seed=2)
    assert sp.math == P.MATH_EXACT
    X, V, st, _ = _run(sp, 10)
    ref, rst = O.run(O.init(_op(sp)), 10)
    assert np.array_equal(X, ref.X) and np.array_equal(V, ref.V) and st.sums == rst.sums


def test_unknown_math_mode_rejected():
    with pytest.raises(P.SpreadError):
        _run(_params((8, 8, 8), math=7), 1)
