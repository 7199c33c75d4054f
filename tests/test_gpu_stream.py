"""Host-streamed mode (somier_stream_*): the paper's
out-of-core cycle -- per step, per chunk: map to (X with halo, V), fused step,
map from -- bit-identical to the CPU oracle for One Buffer (1 slot) and
double buffering (2-3 slots), any chunking."""
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


def _stream_run(sp, steps, chunk, buffers):
    with P.SomierStream(P.Spread([0], 1, sp.n[0] - 2, chunk=chunk), sp, buffers=buffers) as s:
        X, V = s.generate()
        XN = np.zeros_like(X)
        st = None
        for _ in range(steps):
            st = s.step(X, V, XN)
            X, XN = XN, X
        tr = s.traffic()
    return X, V, st, tr


def test_generate_bitwise_equals_oracle_and_resident():
    sp = P.SomierParams(n=(11, 13, 37), seed=8)
    with P.SomierStream(P.Spread([0], 1, 9, chunk=4), sp, buffers=2) as s:
        X, V = s.generate()
    ref = O.init(_op(sp))
    assert np.array_equal(X, ref.X) and not V.any()
    with P.Somier(P.Spread([0], 1, 9), sp) as r:
        Xr, Vr = r.read()
    assert np.array_equal(X, Xr)


@pytest.mark.parametrize("buffers", [1, 2, 3])
@pytest.mark.parametrize("chunk", [3, 5, 100])
def test_stream_steps_bitwise_equal_oracle(buffers, chunk):
    sp = P.SomierParams(n=(14, 17, 40), seed=2)
    X, V, st, tr = _stream_run(sp, 8, chunk, buffers)
    ref, rst = O.run(O.init(_op(sp)), 8)
    assert np.array_equal(X, ref.X) and np.array_equal(V, ref.V)
    assert st.sums == rst.sums and st.vmax2_bits == rst.vmax2_bits and st.centre == rst.centre
    nch = -(-12 // min(chunk, 12))
    assert tr["launches"] == 8 * nch


@pytest.mark.parametrize("kernel", [P.K1_DIRECT, P.K1_MARCH])
def test_stream_matches_resident_and_nonunit_mass(kernel):
    sp = P.SomierParams(n=(20, 9, 33), seed=4, mass=1.7, k_spring=6.0, kernel=kernel)
    X, V, st, _ = _stream_run(sp, 12, 6, 2)
    with P.Somier(P.Spread([0], 1, 18, chunk=7), sp) as r:
        r.step(12)
        Xr, Vr = r.read()
        sr = r.stats()
    assert np.array_equal(X, Xr) and np.array_equal(V, Vr) and st.sums == sr.sums


@pytest.mark.parametrize("devices,chunk,buffers", [([0, 1], 3, 2), ([2, 0, 1], 2, 1), ([0, 1, 2, 3], 5, 3)])
def test_stream_multi_device_logical(devices, chunk, buffers):
    """Listing 10's multi-device round robin (chunk = buffer / ndevices) with
    every list position on its own streams (mapped onto the one GPU)."""
    sp = P.SomierParams(n=(16, 12, 34), seed=5)
    with P.SomierStream(P.Spread(devices, 1, 14, chunk=chunk), sp, buffers=buffers,
                        cuda_devices=[0] * len(devices)) as s:
        X, V = s.generate()
        XN = np.zeros_like(X)
        for _ in range(6):
            st = s.step(X, V, XN)
            X, XN = XN, X
    ref, rst = O.run(O.init(_op(sp)), 6)
    assert np.array_equal(X, ref.X) and np.array_equal(V, ref.V) and st.sums == rst.sums


def test_stream_rejects_aliasing_and_bad_buffers():
    sp = P.SomierParams(n=(8, 8, 8))
    with pytest.raises(P.SpreadError):
        P.SomierStream(P.Spread([0], 1, 6), sp, buffers=0)
    with P.SomierStream(P.Spread([0], 1, 6), sp) as s:
        X, V = s.generate()
        with pytest.raises(P.SpreadError):
            s.step(X, V, X)


@pytest.mark.parametrize("sizes,buffers", [([2, 9, 1, 5], 2), ([17], 1), ([1, 1, 15], 3)])
def test_stream_irregular_chunks(sizes, buffers):
    sp = P.SomierParams(n=(19, 12, 35), seed=4)
    with P.SomierStream(P.Spread.with_sizes([0], 1, 17, sizes), sp, buffers=buffers) as s:
        X, V = s.generate()
        XN = np.zeros_like(X)
        for _ in range(7):
            st = s.step(X, V, XN)
            X, XN = XN, X
    ref, rst = O.run(O.init(_op(sp)), 7)
    assert np.array_equal(X, ref.X) and np.array_equal(V, ref.V)
    assert st.sums == rst.sums


def _pinned_like(a):
    return torch.empty(a.shape, dtype=torch.float64, pin_memory=True).numpy()


@pytest.mark.parametrize("devices,spread_kw,buffers,nsteps", [
    ([0], {"chunk": 3}, 2, 9), ([0], {"chunk": 4}, 1, 10), ([0, 1, 2], {"chunk": 2}, 2, 9),
    ([0, 1], {"sizes": [1, 6, 2, 1, 4]}, 3, 8), ([0, 1, 2, 3], {"chunk": 0}, 2, 5), ([0], {"chunk": 100}, 2, 4)])
def test_stream_run_chunk_level_depend(devices, spread_kw, buffers, nsteps):
    """somier_stream_run: steps chained by per-chunk events only (no barrier per
    step), on pinned host memory so the copies really run asynchronously;
    every step's stats and the final state equal the oracle's bit for bit."""
    n = (16, 13, 37)
    sp = P.SomierParams(n=n, seed=6)
    if "sizes" in spread_kw:
        spread = P.Spread.with_sizes(devices, 1, n[0] - 2, spread_kw["sizes"])
    else:
        spread = P.Spread(devices, 1, n[0] - 2, chunk=spread_kw["chunk"])
    with P.SomierStream(spread, sp, buffers=buffers, cuda_devices=[0] * len(devices)) as s:
        X0, V0 = s.generate()
        X, V, XN = _pinned_like(X0), _pinned_like(V0), _pinned_like(X0)
        X[...] = X0
        V[...] = V0
        XN[...] = np.nan
        stats = s.run(X, V, XN, nsteps)
    final = X if nsteps % 2 == 0 else XN
    ref = O.init(_op(sp))
    for t in range(nsteps):
        ref, rst = O.step(ref)
        assert stats[t].sums == rst.sums and stats[t].vmax2_bits == rst.vmax2_bits and stats[t].step == t + 1
    assert np.array_equal(final, ref.X) and np.array_equal(V, ref.V)


def test_stream_run_equals_steps_and_continues():
    sp = P.SomierParams(n=(12, 10, 33), seed=9)
    with P.SomierStream(P.Spread([0], 1, 10, chunk=3), sp, buffers=2) as s:
        X, V = s.generate()
        XN = np.zeros_like(X)
        s.run(X, V, XN, 3, stats=False)          # X_3 in XN
        st = s.run(XN, V, X, 4)[-1]              # X_7 in XN
        assert st.step == 7
        assert s.run(XN, V, X, 0) == []
        with pytest.raises(P.SpreadError):
            s.run(X, V, X, 2)
    ref, rst = O.run(O.init(_op(sp)), 7)
    assert np.array_equal(XN, ref.X) and np.array_equal(V, ref.V) and st.sums == rst.sums


@pytest.mark.parametrize("devices,spread_kw,buffers,nsteps", [
    ([0], {"chunk": 3}, 2, 8), ([0], {"chunk": 4}, 1, 9), ([0, 1, 2], {"chunk": 2}, 2, 7),
    ([0, 1], {"sizes": [1, 6, 2, 1, 4]}, 3, 6), ([0, 1, 2, 3], {"chunk": 0}, 2, 5), ([0], {"chunk": 100}, 2, 4),
    ([0], {"sizes": [1, 1, 12]}, 2, 3), ([0], {"chunk": 1}, 3, 2)])
def test_stream_run2_two_steps_per_round_trip(devices, spread_kw, buffers, nsteps):
    """somier_stream_run2: two steps per host round trip (K1_TB2 on each chunk
    with X halo 2 and V halo 1 from the host copies, V double-buffered), odd
    step counts end with a one-step launch; chunks of one plane whose halos
    reach two chunks away; the stats after every launch and the final state
    equal the oracle's bit for bit, NaN-filled output buffers leave no trace.
    Stats of every step, both steps of a two-step launch included."""
    n = (16, 13, 37)
    sp = P.SomierParams(n=n, seed=6)
    if "sizes" in spread_kw:
        spread = P.Spread.with_sizes(devices, 1, n[0] - 2, spread_kw["sizes"])
    else:
        spread = P.Spread(devices, 1, n[0] - 2, chunk=spread_kw["chunk"])
    with P.SomierStream(spread, sp, buffers=buffers, cuda_devices=[0] * len(devices)) as s:
        X0, V0 = s.generate()
        X, V, XN, VN = _pinned_like(X0), _pinned_like(V0), _pinned_like(X0), _pinned_like(V0)
        X[...] = X0
        V[...] = V0
        XN[...] = np.nan
        VN[...] = np.nan
        stats = s.run2(X, V, XN, VN, nsteps)
        tr = s.traffic2()
    nl = nsteps // 2 + nsteps % 2
    fX, fV = (X, V) if nl % 2 == 0 else (XN, VN)
    ref = O.init(_op(sp))
    assert len(stats) == nsteps
    for t in range(nsteps):
        ref, rst = O.step(ref)
        assert stats[t].step == t + 1
        assert stats[t].sums == rst.sums and stats[t].vmax2_bits == rst.vmax2_bits and stats[t].centre == rst.centre
    assert np.array_equal(fX, ref.X) and np.array_equal(fV, ref.V)
    plane = 3 * n[1] * n[2] * 8
    assert tr["d2h_bytes"] == 2 * plane * (n[0] - 2) + 4 * plane


def test_stream_run2_matches_run_and_resident():
    """run2 (two steps per round trip) = run (one) = the resident K1_TB2 handle."""
    sp = P.SomierParams(n=(40, 33, 70), seed=9, mass=1.3, k_spring=7.0)
    with P.SomierStream(P.Spread([0], 1, 38, chunk=9), sp, buffers=2) as s:
        X, V = s.generate()
        X2, V2, XN, XN2, VN2 = X.copy(), V.copy(), np.zeros_like(X), np.zeros_like(X), np.zeros_like(V)
        st1 = s.run(X, V, XN, 10)
        st2 = s.run2(X2, V2, XN2, VN2, 10)
        h1 = s.traffic()
        h2 = s.traffic2()
    # run: X_10 in X (even); run2: 5 launches -> (XN2, VN)
    with P.Somier(P.Spread([0], 1, 38), P.SomierParams(n=(40, 33, 70), seed=9, mass=1.3, k_spring=7.0,
                                                       kernel=P.K1_TB2)) as r:
        r.step(10)
        Xr, Vr = r.read()
        sr = r.stats()
    assert st1[-1].sums == st2[-1].sums == sr.sums
    assert np.array_equal(X, Xr) and np.array_equal(V, Vr)
    assert np.array_equal(XN2, Xr) and np.array_equal(VN2, Vr)
    # per node-update, run2 moves about half the host<->device bytes of run
    assert (h2["h2d_bytes"] + h2["d2h_bytes"]) / 2 < 0.6 * (h1["h2d_bytes"] + h1["d2h_bytes"])


@pytest.mark.parametrize("devices,spread_kw,buffers,nsteps,spt", [
    ([0], {"chunk": 3}, 2, 9, 4), ([0], {"chunk": 5}, 1, 10, 8), ([0, 1, 2], {"chunk": 2}, 2, 11, 3),
    ([0, 1], {"sizes": [1, 6, 2, 1, 4]}, 3, 12, 6), ([0], {"chunk": 100}, 2, 7, 5), ([0], {"chunk": 1}, 3, 5, 1),
    ([0, 1, 2, 3], {"chunk": 0}, 2, 13, 13), ([0], {"sizes": [1, 1, 12]}, 2, 6, 2), ([0], {"chunk": 4}, 2, 20, 16)])
def test_stream_run_blocked_s_steps_per_round_trip(devices, spread_kw, buffers, nsteps, spt):
    """somier_stream_run_blocked: s steps per host round trip (halo s, regions
    shrinking two planes per side per K1_TB2 launch, odd s ending with a
    one-step launch, halos reaching several one-plane chunks away, s larger
    than the grid's chunks); every step's stats and the final state equal the
    oracle's bit for bit -- the stats of every step, the intermediate steps of a
    trip (widened launches) included."""
    n = (16, 13, 37)
    sp = P.SomierParams(n=n, seed=6)
    if "sizes" in spread_kw:
        spread = P.Spread.with_sizes(devices, 1, n[0] - 2, spread_kw["sizes"])
    else:
        spread = P.Spread(devices, 1, n[0] - 2, chunk=spread_kw["chunk"])
    with P.SomierStream(spread, sp, buffers=buffers, cuda_devices=[0] * len(devices)) as s:
        X0, V0 = s.generate()
        X, V, XN, VN = _pinned_like(X0), _pinned_like(V0), _pinned_like(X0), _pinned_like(V0)
        X[...] = X0
        V[...] = V0
        XN[...] = np.nan
        VN[...] = np.nan
        stats = s.run_blocked(X, V, XN, VN, nsteps, spt)
    nt = -(-nsteps // spt)
    fX, fV = (X, V) if nt % 2 == 0 else (XN, VN)
    ref = O.init(_op(sp))
    assert len(stats) == nsteps
    for t in range(nsteps):
        ref, rst = O.step(ref)
        assert stats[t].step == t + 1
        assert stats[t].sums == rst.sums and stats[t].vmax2_bits == rst.vmax2_bits
    assert np.array_equal(fX, ref.X) and np.array_equal(fV, ref.V)


def test_stream_run_blocked_matches_run_at_size_and_traffic():
    """A larger grid through 8-step trips (nonunit mass) equals somier_stream_run;
    bytes per node-update fall with the trip length."""
    sp = P.SomierParams(n=(70, 40, 66), seed=2, mass=0.8)
    with P.SomierStream(P.Spread([0], 1, 68, chunk=16), sp, buffers=3) as s:
        X, V = s.generate()
        X2, V2, XN, XN2, VN2 = X.copy(), V.copy(), np.zeros_like(X), np.zeros_like(X), np.zeros_like(V)
        st1 = s.run(X, V, XN, 16)
        st2 = s.run_blocked(X2, V2, XN2, VN2, 16, 8)
        t2 = s.traffic_blocked(2)
        t8 = s.traffic_blocked(8)
        r2 = s.traffic2()
    assert st1[-1].sums == st2[-1].sums and st1[-1].vmax2_bits == st2[-1].vmax2_bits
    assert np.array_equal(X, X2) and np.array_equal(V, V2)  # 2 trips: back in the first buffers
    assert (t8["h2d_bytes"] + t8["d2h_bytes"]) / 8 < 0.5 * (t2["h2d_bytes"] + t2["d2h_bytes"]) / 2
    assert t2["d2h_bytes"] == r2["d2h_bytes"]


def test_stream_fresh_slots_are_zeroed_before_first_copy():
    """Regression: the slots' zeroing (cudaMemset, legacy stream) must finish
    before the handle's non-blocking streams copy the first chunk in -- else it
    could wipe the first planes of a chunk mapped right after creation (a wide
    cross-section makes the memset long enough to lose that race)."""
    n = (24, 512, 512)
    sp = P.SomierParams(n=n, seed=8)
    want = None
    for rep in range(3):
        for spt, buffers in ((2, 1), (4, 1), (2, 3)):
            with P.SomierStream(P.Spread([0], 1, n[0] - 2, chunk=22 if rep else 8), sp, buffers=buffers) as s:
                X, V = s.generate()
                XN, VN = np.zeros_like(X), np.zeros_like(V)
                st = s.run_blocked(X, V, XN, VN, 4, spt)[-1]
                fX, fV = (X, V) if (-(-4 // spt)) % 2 == 0 else (XN, VN)
            key = (st.sums, st.vmax2_bits, fX[:, :6].tobytes(), fV[:, :6].tobytes())
            want = want or key
            assert key == want


def test_stream_modes_alternate_on_one_handle():
    """One-step cycles and blocked trips on the same handle (the two kinds of
    device slots are swapped in and out): the state carries through bit for bit."""
    n = (18, 11, 35)
    sp = P.SomierParams(n=n, seed=12)
    with P.SomierStream(P.Spread([0], 1, n[0] - 2, chunk=5), sp, buffers=2) as s:
        X, V = s.generate()
        XN, VN = np.zeros_like(X), np.zeros_like(V)
        s.run(X, V, XN, 3)                     # X_3 in XN, V in place
        X, XN = XN, X
        s.run_blocked(X, V, XN, VN, 4, 2)      # 2 trips: back in (X, V)
        s.run(X, V, XN, 1)                     # X_8 in XN
        X, XN = XN, X
        st = s.run2(X, V, XN, VN, 3)[-1]       # 2 launches: back in (X, V)
    ref, rst = O.run(O.init(_op(sp)), 11)
    assert np.array_equal(X, ref.X) and np.array_equal(V, ref.V)
    assert st.sums == rst.sums and st.step == 11


@pytest.mark.parametrize("mode", ["run", "run2", "blocked4"])
def test_stream_non_unit_mass_prestressed_vs_oracle(mode):
    """The host-streamed paths (one-step kernel, K1_TB2 two steps per trip, s
    steps per trip) at M != 1 and rest length != spacing, directly against the
    oracle: every step's stats and the final state bitwise."""
    n, nsteps = (15, 11, 34), 6
    sp = P.SomierParams(n=n, seed=12, mass=0.7, spacing=1.25, rest_len=1.0, k_spring=4.0, dt=2e-3, amplitude=0.1)
    with P.SomierStream(P.Spread([0, 1], 1, n[0] - 2, chunk=3), sp, buffers=2, cuda_devices=[0, 0]) as s:
        X0, V0 = s.generate()
        X, V, XN, VN = _pinned_like(X0), _pinned_like(V0), _pinned_like(X0), _pinned_like(V0)
        X[...] = X0
        V[...] = V0
        if mode == "run":
            stats = s.run(X, V, XN, nsteps)
            fX, fV = (X, V)
        elif mode == "run2":
            stats = s.run2(X, V, XN, VN, nsteps)
            fX, fV = (XN, VN)  # 3 launches
        else:
            stats = s.run_blocked(X, V, XN, VN, nsteps, 4)
            fX, fV = (X, V)  # 2 trips
    ref = O.init(_op(sp))
    for t in range(nsteps):
        ref, rst = O.step(ref)
        assert stats[t].sums == rst.sums and stats[t].vmax2_bits == rst.vmax2_bits, t
    assert np.array_equal(fX, ref.X) and np.array_equal(fV, ref.V)
