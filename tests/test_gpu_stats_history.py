"""Per-step stats on the GPU: the "centers" kernel runs after EVERY time step
(reading S8), so every kernel -- K1_TB2's two-step
launches included -- computes the centre and vmax of every state, and the
handle exposes them (somier_stats_history, a device-side ring the kernels
index from a device step counter, so graph replays need no per-step
arguments). Each step's stats must equal the oracle's `centers` of that state
bit for bit, on one chunk and on multi-position spreads, for any split of the
step calls."""
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


def _oracle_history(sp, nsteps):
    """[(state, stats)] for states 0 .. nsteps."""
    s = O.init(_op(sp))
    out = [(s, O.centers(s))]
    for _ in range(nsteps):
        s, st = O.step(s)
        out.append((s, st))
    return out


def _same(a, b):
    return a.sums == b.sums and a.vmax2_bits == b.vmax2_bits and a.centre == b.centre and a.vmax == b.vmax


@pytest.mark.parametrize("kernel", [P.K1_TB2, P.K1_MARCH2, P.K1_MARCH, P.K1_DIRECT])
@pytest.mark.parametrize("devices,chunk", [([0], 0), ([0], 5), ([0, 1], 0), ([2, 0, 1], 4)])
@pytest.mark.parametrize("splits", [[2, 2, 2, 2, 2, 10], [20], [1, 5, 2, 11, 1], [3, 3, 3, 3, 3, 3, 2]])
def test_every_step_bitwise(kernel, devices, chunk, splits):
    n = (19, 17, 40)
    sp = P.SomierParams(n=n, seed=5, kernel=kernel)
    total = sum(splits)
    ref = _oracle_history(sp, total)
    spread = P.Spread(devices, 1, n[0] - 2, chunk=chunk)
    with P.Somier(spread, sp, cuda_devices=[0] * len(devices)) as s:
        h0 = s.stats_history(0, 1)[0]
        assert h0.step == 0 and _same(h0, ref[0][1])
        done = 0
        for k in splits:
            s.step(k)
            done += k
            hist = s.stats_history(0, done + 1)
            for t, st in enumerate(hist):
                assert st.step == t
                assert _same(st, ref[t][1]), "stats of step %d differ (kernel %d, after %d steps)" % (t, kernel, done)
            assert _same(s.stats(), ref[done][1])
        X, V = s.read()
    assert np.array_equal(X, ref[total][0].X) and np.array_equal(V, ref[total][0].V)


@pytest.mark.parametrize("kernel", [P.K1_TB2, P.K1_MARCH2])
def test_tb2_non_unit_mass_prestressed_vs_oracle(kernel):
    """K1_TB2's kUnitMass=false instantiation (and the force's use of L != spacing)
    against the oracle directly, every step's stats included."""
    n = (14, 15, 66)
    sp = P.SomierParams(n=n, seed=8, mass=2.5, spacing=1.25, rest_len=1.0, k_spring=7.0, dt=2e-3, amplitude=0.1,
                        kernel=kernel)
    ref = _oracle_history(sp, 24)
    with P.Somier(P.Spread([0], 1, n[0] - 2), sp) as s:
        assert s.kernel_in_use == kernel
        s.step(24)
        hist = s.stats_history(0, 25)
        X, V = s.read()
    assert np.array_equal(X, ref[24][0].X) and np.array_equal(V, ref[24][0].V)
    for t in range(25):
        assert _same(hist[t], ref[t][1])


def test_history_window_and_reset_on_load():
    """The ring keeps the last STATS_HISTORY steps since init/load; steps outside
    it are EINVAL; a load restarts the history at the current step."""
    n = (10, 9, 12)
    sp = P.SomierParams(n=n, seed=2, kernel=P.K1_TB2)
    total = P.STATS_HISTORY + 30
    ref = _oracle_history(sp, total)
    with P.Somier(P.Spread([0], 1, n[0] - 2), sp) as s:
        s.step(total)
        lo = total - P.STATS_HISTORY + 1
        hist = s.stats_history(lo, P.STATS_HISTORY)
        for i, st in enumerate(hist):
            assert st.step == lo + i and _same(st, ref[lo + i][1])
        with pytest.raises(P.SpreadError):
            s.stats_history(lo - 1, 1)
        with pytest.raises(P.SpreadError):
            s.stats_history(total, 2)
        X, V = s.read()
        s.load(X, V)
        with pytest.raises(P.SpreadError):
            s.stats_history(total - 1, 1)
        assert _same(s.stats_history(total, 1)[0], ref[total][1])
        s.step(3)
        st = ref[total][0]
        for t in range(1, 4):
            st, rst = O.step(st)
            assert _same(s.stats_history(total + t, 1)[0], rst)


def test_history_in_graph_replays():
    """K1_TB2 graph replays (4 steps per replay) keep writing the right ring
    slots: the slot comes from the device step word, not a baked argument."""
    n = (70, 20, 33)
    sp = P.SomierParams(n=n, seed=4, kernel=P.K1_TB2)
    ref = _oracle_history(sp, 41)
    with P.Somier(P.Spread([0], 1, n[0] - 2), sp) as s:
        s.step(40)
        s.step(1)
        hist = s.stats_history(0, 42)
    for t in range(42):
        assert _same(hist[t], ref[t][1])


@pytest.mark.parametrize("n1", [3, 21, 22, 23, 43, 44, 45, 66])
@pytest.mark.parametrize("n2", [3, 31, 32, 33, 62])
def test_tb2_tile_edges_every_step(n1, n2):
    """K1_TB2 counts step t+1's nodes over R1 rows [jq - 1, jq + 21) (a
    partition of the j axis shifted by one row against the owned tiles) and
    drops ring / k-face columns per thread: cross-sections whose n1 is a
    multiple of the 22-row tile (one more tile row), one below or above it, and
    k extents around the 30-column tiles -- every step's stats and the state
    bit for bit vs the oracle."""
    n = (9, n1, n2)
    sp = P.SomierParams(n=n, seed=11, kernel=P.K1_TB2)
    ref = _oracle_history(sp, 6)
    with P.Somier(P.Spread([0], 1, n[0] - 2), sp) as s:
        assert s.kernel_in_use == P.K1_TB2
        s.step(6)
        hist = s.stats_history(0, 7)
        X, V = s.read()
    assert np.array_equal(X, ref[6][0].X) and np.array_equal(V, ref[6][0].V)
    for t in range(7):
        assert _same(hist[t], ref[t][1]), "step %d" % t
