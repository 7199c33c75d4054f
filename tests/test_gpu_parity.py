"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bar (BASELINE.json north_star): positions and velocities within
1e-10 normwise relative error after 100 steps. The kernels use explicit IEEE
round-to-nearest intrinsics and no contraction, exactly like the oracle, so the
tests also assert the stronger property the design delivers: bit-identical X, V
and stats. Partitioned runs (any chunk size / device order) must be
bit-identical to the single-chunk run.
"""
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


def _params(n, seed=1, kernel=P.K1_AUTO, **kw):
    return P.SomierParams(n=tuple(n), seed=seed, kernel=kernel, **kw)


def _oracle_params(sp: "P.SomierParams"):
    return O.Params(n=sp.n, spacing=sp.spacing, rest_len=sp.rest_len, k_spring=sp.k_spring, mass=sp.mass,
                    dt=sp.dt, amplitude=sp.amplitude, seed=sp.seed)


def _run_gpu(sp, steps, devices=(0,), chunk=0):
    spread = P.Spread(list(devices), 1, sp.n[0] - 2, chunk=chunk)
    with P.Somier(spread, sp) as s:
        s.step(steps)
        st = s.stats()
        X, V = s.read()
    return X, V, st


def _rel(a, b):
    den = np.max(np.abs(b))
    return np.max(np.abs(a - b)) / den if den > 0 else np.max(np.abs(a - b))


def _assert_parity(X, V, st, ref, rst, bitwise=True):
    x0 = O.init(ref.p).X
    assert _rel(X, ref.X) <= 1e-10
    assert _rel(X - x0, ref.X - x0) <= 1e-10     # displacement: the stricter reading S12
    assert _rel(V, ref.V) <= 1e-10
    if bitwise:
        assert np.array_equal(X, ref.X), "X differs bitwise from the oracle"
        assert np.array_equal(V, ref.V), "V differs bitwise from the oracle"
        assert st.sums == rst.sums and st.vmax2_bits == rst.vmax2_bits
        assert st.centre == rst.centre and st.vmax == rst.vmax


@pytest.mark.parametrize("kernel", [P.K1_DIRECT, P.K1_MARCH, P.K1_MARCH2, P.K1_TB2])
@pytest.mark.parametrize("n", [(16, 16, 16), (17, 9, 33), (3, 3, 3), (5, 40, 70)])
def test_initial_state_bitwise(n, kernel):
    sp = _params(n, seed=2, kernel=kernel)
    X, V, st = _run_gpu(sp, 0)
    ref = O.init(_oracle_params(sp))
    assert np.array_equal(X, ref.X) and np.array_equal(V, ref.V)
    rst = O.centers(ref)
    assert st.sums == rst.sums and st.centre == rst.centre and st.vmax2_bits == rst.vmax2_bits


@pytest.mark.parametrize("kernel", [P.K1_DIRECT, P.K1_MARCH, P.K1_MARCH2, P.K1_TB2])
@pytest.mark.parametrize("seed", [1, 2, 3])
def test_16cube_10_steps(seed, kernel):
    """configs[0]: Somier 16^3, fp64, 10 steps."""
    sp = _params((16, 16, 16), seed=seed, kernel=kernel)
    X, V, st = _run_gpu(sp, 10)
    ref, rst = O.run(O.init(_oracle_params(sp)), 10)
    _assert_parity(X, V, st, ref, rst)


@pytest.mark.parametrize("kernel", [P.K1_DIRECT, P.K1_MARCH, P.K1_MARCH2, P.K1_TB2])
@pytest.mark.parametrize("n", [(17, 9, 33), (9, 33, 17), (33, 17, 9), (6, 131, 70), (4, 5, 260)])
def test_ragged_shapes_30_steps(n, kernel):
    """Shapes spanning several tiles with ragged tails in every dimension."""
    sp = _params(n, seed=5, kernel=kernel)
    X, V, st = _run_gpu(sp, 30)
    ref, rst = O.run(O.init(_oracle_params(sp)), 30)
    _assert_parity(X, V, st, ref, rst)


@pytest.mark.parametrize("kernel", [P.K1_DIRECT, P.K1_MARCH, P.K1_MARCH2, P.K1_TB2])
def test_128cube_100_steps(kernel):
    """configs[1]: Somier 128^3, 100 steps, 1 GPU vs the CPU oracle."""
    sp = _params((128, 128, 128), seed=1, kernel=kernel)
    X, V, st = _run_gpu(sp, 100)
    ref, rst = _oracle_128()
    _assert_parity(X, V, st, ref, rst)


_CACHE = {}


def _oracle_128():
    if "128" not in _CACHE:
        sp = _params((128, 128, 128), seed=1)
        _CACHE["128"] = O.run(O.init(_oracle_params(sp)), 100)
    return _CACHE["128"]


def test_non_unit_mass_and_spacing():
    sp = _params((12, 14, 18), seed=7, mass=2.5, spacing=0.75, rest_len=0.8, k_spring=3.0, dt=2e-3, amplitude=0.1)
    X, V, st = _run_gpu(sp, 40)
    ref, rst = O.run(O.init(_oracle_params(sp)), 40)
    _assert_parity(X, V, st, ref, rst)


@pytest.mark.parametrize("chunk", [1, 2, 3, 5, 7, 13, 100])
def test_virtual_devices_bit_identical(chunk):
    """Several chunks on one device (static round-robin over a 1-device list):
    halos move by the fused in-kernel stores; result bit-identical to 1 chunk."""
    sp = _params((16, 12, 20), seed=3)
    X1, V1, s1 = _run_gpu(sp, 25)
    Xc, Vc, sc = _run_gpu(sp, 25, devices=(0,), chunk=chunk)
    assert np.array_equal(X1, Xc) and np.array_equal(V1, Vc)
    assert s1.sums == sc.sums and s1.vmax2_bits == sc.vmax2_bits and s1.centre == sc.centre


def test_rest_lattice_stays_exactly_at_rest_on_gpu():
    """C4 on the GPU: amplitude 0 -> every spring at rest length -> bitwise fixed point."""
    sp = _params((9, 10, 11), amplitude=0.0)
    X0, V0, _ = _run_gpu(sp, 0)
    X, V, st = _run_gpu(sp, 50, chunk=3)
    assert np.array_equal(X, X0) and not V.any()
    assert st.centre == (0.0, 0.0, 0.0) and st.vmax == 0.0


def _mirror(n, axis, seed):
    rng = np.random.default_rng(seed)
    sp0 = O.Params(n=n, amplitude=0.0)
    s = O.init(sp0)
    X, V = s.X, np.zeros_like(s.X)
    sign = np.ones((3, 1, 1, 1))
    sign[axis] = -1
    m = n[axis]
    for arr, amp in ((X, 0.05), (V, 0.01)):
        d = rng.uniform(-amp, amp, size=X.shape)
        d[:, [0, -1], :, :] = 0
        d[:, :, [0, -1], :] = 0
        d[:, :, :, [0, -1]] = 0
        lower = np.take(d, range(m // 2), axis=1 + axis)
        idx = [slice(None)] * 4
        idx[1 + axis] = slice(m - m // 2, m)
        d[tuple(idx)] = np.flip(lower, axis=1 + axis) * sign
        if m % 2:
            idx[1 + axis] = m // 2
            d[axis][tuple(idx[1:])] = 0
        arr += d
    return X, V, sign


@pytest.mark.parametrize("axis", [0, 1, 2])
def test_mirror_symmetry_bitwise_on_gpu(axis):
    """C5 on the GPU through somier_load: odd displacement stays exactly odd."""
    n = (8, 7, 9)
    X0, V0, sign = _mirror(n, axis, seed=axis)
    sp = _params(n)
    spread = P.Spread([0], 1, n[0] - 2, chunk=2)
    with P.Somier(spread, sp) as s:
        s.load(X0, V0)
        s.step(100)
        X, V = s.read()
        st = s.stats()
    flip = lambda a: np.flip(a, axis=1 + axis)
    assert np.array_equal(flip(X) * sign, X) and np.array_equal(flip(V) * sign, V)
    assert st.centre[axis] == 0.0
    # and it is the oracle's trajectory, bit for bit
    ref = O.State(_oracle_params(sp), *(np.ascontiguousarray(a) for a in (*X0, *V0)))
    ref, rst = O.run(ref, 100)
    assert np.array_equal(X, ref.X) and np.array_equal(V, ref.V)


def test_load_read_roundtrip_and_continue():
    sp = _params((10, 11, 12), seed=4)
    rng = np.random.default_rng(0)
    spread = P.Spread([0], 1, 8, chunk=3)
    with P.Somier(spread, sp) as s:
        X0, V0 = s.read()
        X0 = X0 + rng.uniform(-0.01, 0.01, X0.shape) * 0  # unchanged faces
        V0 = V0.copy()
        V0[:, 1:-1, 1:-1, 1:-1] = rng.uniform(-0.02, 0.02, (3, 8, 9, 10))
        s.load(X0, V0)
        X1, V1 = s.read()
        assert np.array_equal(X1, X0) and np.array_equal(V1, V0)
        st0 = s.stats()
        ref0 = O.State(_oracle_params(sp), *(np.ascontiguousarray(a) for a in (*X0, *V0)))
        assert st0.sums == O.centers(ref0).sums
        s.step(7)
        X2, V2 = s.read()
        st = s.stats()
    ref, rst = O.run(ref0, 7)
    assert np.array_equal(X2, ref.X) and np.array_equal(V2, ref.V) and st.sums == rst.sums


def test_stats_every_step_matches_oracle():
    sp = _params((12, 12, 12), seed=9)
    spread = P.Spread([0], 1, 10, chunk=4)
    ref = O.init(_oracle_params(sp))
    with P.Somier(spread, sp) as s:
        for t in range(5):
            s.step(1)
            st = s.stats()
            ref, rst = O.step(ref)
            assert st.step == t + 1
            assert st.sums == rst.sums and st.vmax2_bits == rst.vmax2_bits and st.centre == rst.centre


def test_errors_are_reported():
    sp = _params((10, 10, 10))
    with pytest.raises(P.SpreadError) as e:
        P.Somier(P.Spread([0], 0, 10), sp)         # range must be (1 : n0-2)
    assert e.value.status == -1
    with pytest.raises(P.SpreadError) as e:
        P.Somier(P.Spread([0, 99], 1, 8), sp)      # no device 99
    assert e.value.status == -2
    with pytest.raises(P.SpreadError):
        P.Somier(P.Spread([0], 1, 8), _params((10, 10, 10), mass=0.0))


def test_launch_count_and_footprint():
    sp = _params((34, 20, 40))
    spread = P.Spread([0], 1, 32, chunk=8)
    with P.Somier(spread, sp) as s:
        assert s.local_chunks == 4
        s.step(3)
        s.sync()
        assert s.launches == 12
        assert s.device_bytes >= (2 * 34 + 32) * 3 * 20 * 40 * 8


@pytest.mark.parametrize("kernel", [P.K1_DIRECT, P.K1_MARCH, P.K1_MARCH2, P.K1_TB2])
@pytest.mark.parametrize("K", [0.0, -2.0])
def test_zero_and_negative_stiffness_signed_zeros(K, kernel):
    """K <= 0 makes K*(d-L) = -0 possible; -0/d must stay -0 (the K > 0 fast
    path drops that select). Bitwise vs the oracle, signed zeros included."""
    sp = _params((9, 10, 33), seed=6, kernel=kernel, k_spring=K)
    X, V, st = _run_gpu(sp, 12)
    ref, rst = O.run(O.init(_oracle_params(sp)), 12)
    assert np.array_equal(X.view(np.uint64), ref.X.view(np.uint64))
    assert np.array_equal(V.view(np.uint64), ref.V.view(np.uint64))
