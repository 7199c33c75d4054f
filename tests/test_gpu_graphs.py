"""CUDA-graph replay of (even, odd) step pairs: any split of
the step count, starting on either parity, gives the oracle's bits; launch
counting stays exact; SOMIER_NO_GRAPH=1 (eager launches) gives the same bits."""
import os

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


@pytest.mark.parametrize("splits", [(13,), (3, 4, 1, 5), (1, 1, 11), (2, 2, 2, 7)])
@pytest.mark.parametrize("chunk", [0, 4])
def test_graph_splits_bitwise(splits, chunk):
    sp = P.SomierParams(n=(12, 10, 36), seed=3, kernel=P.K1_MARCH2)  # graphs replay one-step kernels
    with P.Somier(P.Spread([0], 1, 10, chunk=chunk), sp) as s:
        for k in splits:
            s.step(k)
        X, V = s.read()
        st = s.stats()
        nloc = s.local_chunks
        assert s.launches == 13 * nloc
    ref, rst = O.run(O.init(O.Params(n=sp.n, seed=3)), 13)
    assert np.array_equal(X, ref.X) and np.array_equal(V, ref.V) and st.sums == rst.sums


def test_eager_and_graph_identical(monkeypatch):
    sp = P.SomierParams(n=(16, 16, 40), seed=9, kernel=P.K1_MARCH2)
    outs = []
    for env in ("0", "1"):
        monkeypatch.setenv("SOMIER_NO_GRAPH", env)
        with P.Somier(P.Spread([0], 1, 14, chunk=5), sp) as s:
            s.step(20)
            outs.append(s.read())
    assert np.array_equal(outs[0][0], outs[1][0]) and np.array_equal(outs[0][1], outs[1][1])


def _tb2_launches(splits):
    """K1_TB2 launch rule (somier_step): pairs of steps, then a leftover single
    step (the same kernel in one-step mode), whatever the start parity."""
    return sum(k // 2 + k % 2 for k in splits)


@pytest.mark.parametrize("chunk", [0, 4])
@pytest.mark.parametrize("splits", [(13,), (3, 4, 1, 5), (1, 1, 11), (2, 2, 2, 7), (1, 12), (5, 9, 4, 6)])
def test_tb2_splits_bitwise(splits, chunk):
    """K1_TB2 (two steps per launch, AUTO on large single-chunk grids): any split
    of the step count, on either parity, gives the oracle's bits, stats
    included -- through the graph replays of two pairs (keyed by buffer and
    step parity) and the eager pairs / single steps around them; chunk 4: three
    chunks on one stream (deep-halo stores inside the graph)."""
    sp = P.SomierParams(n=(12, 10, 36), seed=3, kernel=P.K1_TB2)
    with P.Somier(P.Spread([0], 1, 10, chunk=chunk), sp) as s:
        assert s.kernel_in_use == P.K1_TB2
        for k in splits:
            s.step(k)
            st = s.stats()
            ref, rst = O.run(O.init(O.Params(n=sp.n, seed=3)), s.step_count)
            assert st.sums == rst.sums and st.vmax2_bits == rst.vmax2_bits, (splits, k)
        X, V = s.read()
        assert s.launches == _tb2_launches(splits) * s.local_chunks
    assert np.array_equal(X, ref.X) and np.array_equal(V, ref.V)


def test_tb2_eager_and_graph_identical(monkeypatch):
    sp = P.SomierParams(n=(20, 18, 40), seed=9, kernel=P.K1_TB2)
    outs = []
    for env in ("0", "1"):
        monkeypatch.setenv("SOMIER_NO_GRAPH", env)
        with P.Somier(P.Spread([0], 1, 18, chunk=6), sp) as s:
            s.step(3)
            s.step(22)
            outs.append(s.read() + (s.stats().sums,))
    assert np.array_equal(outs[0][0], outs[1][0]) and np.array_equal(outs[0][1], outs[1][1])
    assert outs[0][2] == outs[1][2]


def test_auto_kernel_resolution():
    big = P.SomierParams(n=(200, 200, 200), seed=3)  # 8e6 nodes: K1_TB2's range
    with P.Somier(P.Spread([0], 1, 198), big) as s:
        assert s.kernel_in_use == P.K1_TB2
    tall = P.SomierParams(n=(320, 200, 200), seed=3)
    with P.Somier(P.Spread([0], 1, 318, chunk=159), tall) as s:
        assert s.kernel_in_use == P.K1_TB2  # two chunks of 159 planes x 200^2 nodes: K1_TB2 with deep halos
    with P.Somier(P.Spread([0], 1, 198, chunk=40), big) as s:
        assert s.kernel_in_use == P.K1_MARCH2  # a chunk of 38 planes (1.5e6 nodes): below TB2's range
    sp = P.SomierParams(n=(12, 10, 36), seed=3)
    with P.Somier(P.Spread([0], 1, 10), sp) as s:
        assert s.kernel_in_use == P.K1_MARCH2  # small grid: TB2's tiles fill too few waves
    with P.Somier(P.Spread([0], 1, 10), P.SomierParams(n=(12, 10, 36), kernel=P.K1_MARCH)) as s:
        assert s.kernel_in_use == P.K1_MARCH


def test_launch_timing_instrumentation_keeps_results():
    """somier_set_timing: every launch bracketed by events (graph replay off);
    take_timing reports one record per launch with plausible times, and the
    results stay bit-identical to an untimed run."""
    n = (40, 24, 37)
    sp = P.SomierParams(n=n, seed=5, kernel=P.K1_TB2)
    with P.Somier(P.Spread([0, 1], 1, n[0] - 2), sp, cuda_devices=[0, 0]) as s:
        s.set_timing(True)
        s.step(9)
        t = s.take_timing()
        s.set_timing(False)
        s.step(3)
        X, V = s.read()
        st = s.stats()
    assert t["launches"] == 2 * 5  # two positions x (4 two-step + 1 one-step launches)
    assert t["kernel_ms"] > 0 and t["wait_ms"] >= 0 and t["kernel_max_ms"] <= t["kernel_ms"]
    with P.Somier(P.Spread([0], 1, n[0] - 2), sp) as r:
        r.step(12)
        Xr, Vr = r.read()
        sr = r.stats()
    assert np.array_equal(X, Xr) and np.array_equal(V, Vr) and st.sums == sr.sums
