"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (single chunk, K1 AUTO): single nodes checked bit for bit through their
light cone (a node after S steps depends only on initial values within
distance S, so the oracle on a window reaching S+1 beyond it reproduces it
exactly -- pinned in tests/test_oracle_pins.py), plus size-independent
properties (rest lattice fixed point, centre exactly 0)."""
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


def _samples(n, rng, count):
    out = [(1, 1, 1), (n[0] - 2, n[1] - 2, n[2] - 2), (n[0] // 2, 1, n[2] - 2), (1, n[1] // 2, n[2] // 2),
           (n[0] // 2, n[1] // 2, 31), (n[0] // 2, 15, 32), (65, 16, 33), (64, 17, 96),
           # K1_TB2 tile / segment borders (owned tiles 30 x 22 from k = 1, j = 0; at 512^3 five segments of
           # 102 planes from i = 1, at 1024^3 seven of 146)
           (65, 22, 30), (64, 21, 29), (129, 44, 60), (n[0] - 2, n[1] - 2, 30), (102, 23, 31), (103, 22, 1),
           (104, 66, 61), (147, 88, 91), (148, 43, 90)]
    while len(out) < count:
        out.append(tuple(int(rng.integers(1, n[d] - 1)) for d in range(3)))
    return out


def _check_nodes(n, steps, count, seed=42, kernel=P.K1_AUTO, devices=(0,), extra=()):
    sp = P.SomierParams(n=n, seed=seed, kernel=kernel)
    op = O.Params(n=n, seed=seed)
    rng = np.random.default_rng(7)
    nodes = list(extra) + _samples(n, rng, count)
    with P.Somier(P.Spread(list(devices), 1, n[0] - 2), sp, cuda_devices=[0] * len(devices)) as s:
        if kernel == P.K1_AUTO:
            assert s.kernel_in_use == P.K1_TB2
        s.step(steps)
        got = {}
        for c in nodes:
            X, V = s.read_planes(c[0], 1)
            got[c] = (X[:, 0, c[1], c[2]].copy(), V[:, 0, c[1], c[2]].copy())
    for c in nodes:
        lo = [max(0, c[d] - steps - 1) for d in range(3)]
        hi = [min(n[d], c[d] + steps + 2) for d in range(3)]
        win, _ = O.run(O.init_window(op, lo, [hi[d] - lo[d] for d in range(3)]), steps)
        r = tuple(c[d] - lo[d] for d in range(3))
        want_x = win.X[(slice(None),) + r]
        want_v = win.V[(slice(None),) + r]
        assert np.array_equal(got[c][0], want_x), (c, got[c][0], want_x)
        assert np.array_equal(got[c][1], want_v), (c, got[c][1], want_v)


def test_512cube_bench_config_sampled_nodes_bitwise():
    """configs[3] (the bench workload, K1 AUTO = K1_TB2): 512^3, 24 steps, 16 nodes."""
    _check_nodes((512, 512, 512), 24, 16)


def test_512cube_two_positions_deep_halo_sampled_nodes_bitwise():
    """The bench's N = 2 layout on one GPU: 512^3 over devices(0,1) (two chunks
    of 255 planes, K1 AUTO = K1_TB2 with the two-plane halo exchange between
    list positions), 13 steps (six two-step launches and one single step);
    nodes on both sides of the chunk boundary and its deep halo planes."""
    edge = [(254, 40, 77), (255, 300, 13), (256, 5, 500), (257, 255, 256), (253, 1, 1), (258, 510, 510)]
    _check_nodes((512, 512, 512), 13, 10, devices=(0, 1), extra=edge)


def test_512cube_march2_kernel_sampled_nodes_bitwise():
    """The one-step kernel multi-chunk / multi-GPU runs use, at the bench size."""
    _check_nodes((512, 512, 512), 24, 12, kernel=P.K1_MARCH2)


def test_512cube_march_kernel_sampled_nodes_bitwise():
    _check_nodes((512, 512, 512), 12, 6, kernel=P.K1_MARCH)


def test_1024cube_sampled_nodes_bitwise():
    """configs[4] grid (77 GB on one GPU): 1024^3, 10 steps, 8 nodes."""
    _check_nodes((1024, 1024, 1024), 10, 8)


def test_1024cube_eight_positions_configs4_layout_sampled_nodes_bitwise():
    """configs[4]'s layout on one GPU: 1024^3 spread over devices(0..7) (eight
    chunks of 128 planes and one of 126, K1 AUTO = K1_TB2 with the deep-halo
    exchange between positions), 5 steps (two two-step launches and one single
    step); nodes on both sides of chunk boundaries."""
    edge = [(128, 500, 3), (129, 1, 1022), (130, 700, 700), (256, 31, 30), (257, 1022, 1022), (897, 511, 512),
            (896, 2, 64), (1022, 640, 333)]
    _check_nodes((1024, 1024, 1024), 5, 6, devices=tuple(range(8)), extra=edge)


def test_512cube_rest_lattice_fixed_point_and_zero_centre():
    sp = P.SomierParams(n=(512, 512, 512), amplitude=0.0)
    with P.Somier(P.Spread([0], 1, 510), sp) as s:
        X0, _ = s.read_planes(200, 3)
        s.step(6)
        st = s.stats()
        X1, V1 = s.read_planes(200, 3)
    assert np.array_equal(X0, X1) and not V1.any()
    assert st.centre == (0.0, 0.0, 0.0) and st.vmax == 0.0 and st.nodes == 512 ** 3


def test_512cube_full_state_and_every_step_stats_vs_full_oracle():
    """The bench configuration at full size against the oracle run on the whole
    512^3 grid (the -fopenmp build, bit-identical to the sequential oracle:
    tests/test_oracle_omp.py): centre sums and vmax of each of 4 steps (two
    K1_TB2 launches, both steps of each) and every element of the final X and V
    bit for bit."""
    n, steps = (512, 512, 512), 4
    sp = P.SomierParams(n=n, seed=42)
    with P.Somier(P.Spread([0], 1, n[0] - 2), sp) as s:
        assert s.kernel_in_use == P.K1_TB2
        s.step(steps)
        hist = s.stats_history(1, steps)
        X, V = s.read()
    st = O.init(O.Params(n=n, seed=42))
    for t in range(steps):
        st, ost, _, _ = O.run_timed(st, 1, omp=True)
        assert hist[t].sums == ost.sums and hist[t].vmax2_bits == ost.vmax2_bits, t + 1
    for c, (xo, vo) in enumerate(zip((st.x, st.y, st.z), (st.vx, st.vy, st.vz))):
        assert np.array_equal(X[c], xo), "X component %d" % c
        assert np.array_equal(V[c], vo), "V component %d" % c


def test_256cube_100_steps_spread_2_and_4_vs_full_oracle():
    """BASELINE configs[2] -- 256^3, 100 steps, spread over 2 and 4 list
    positions (logical devices on one GPU: the cross-position exchange runs
    exactly as between GPUs) -- every element of X and V and every step's
    stats against the whole-grid oracle (-fopenmp build), bit for bit."""
    n, steps = (256, 256, 256), 100
    op = O.Params(n=n, seed=42)
    st = O.init(op)
    ref = []
    for _ in range(steps):
        st, ost, _, _ = O.run_timed(st, 1, omp=True)
        ref.append(ost)
    for devs in ([0, 1], [0, 1, 2, 3]):
        sp = P.SomierParams(n=n, seed=42)
        with P.Somier(P.Spread(devs, 1, n[0] - 2), sp, cuda_devices=[0] * len(devs)) as s:
            s.step(steps)
            hist = s.stats_history(steps - P.STATS_HISTORY + 1, P.STATS_HISTORY) if steps > P.STATS_HISTORY \
                else s.stats_history(1, steps)
            X, V = s.read()
        first = steps - len(hist) + 1
        for i, h in enumerate(hist):
            r = ref[first - 1 + i]
            assert h.sums == r.sums and h.vmax2_bits == r.vmax2_bits, (devs, first + i)
        for c, (xo, vo) in enumerate(zip((st.x, st.y, st.z), (st.vx, st.vy, st.vz))):
            assert np.array_equal(X[c], xo) and np.array_equal(V[c], vo), (devs, c)
