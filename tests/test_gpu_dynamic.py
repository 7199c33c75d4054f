"""spread_schedule(dynamic, chunk) -- the paper's future work against load
imbalance: in the host-streamed Somier each chunk goes to
whichever list position frees a buffer slot first. The state and every step's
stats must be bit-identical to the oracle (and so to the static schedule)
whatever the assignment; with one position deliberately slowed
(somier_stream_set_delay) the other takes more of the chunks. The generic
spread loops (stencil3, reduce) accept the dynamic schedule too."""
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


def _pinned(shape):
    return torch.zeros(shape, dtype=torch.float64, pin_memory=True).numpy()


@pytest.mark.parametrize("devices,chunk,buffers,delay_pos", [([0, 1], 3, 2, 1), ([0, 1, 2], 2, 2, 0),
                                                             ([0, 1], 1, 3, None), ([0], 4, 2, None)])
@pytest.mark.parametrize("mode", ["run", "run2", "blocked3"])
def test_dynamic_stream_bitwise(devices, chunk, buffers, delay_pos, mode):
    n, nsteps = (20, 13, 37), 7
    sp = P.SomierParams(n=n, seed=4)
    spread = P.Spread(devices, 1, n[0] - 2, chunk=chunk, sched=P.SCHED_DYNAMIC)
    assert spread.dynamic
    with P.SomierStream(spread, sp, buffers=buffers, cuda_devices=[0] * len(devices)) as s:
        if delay_pos is not None:
            s.set_delay(delay_pos, 200_000)
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
        counts = s.chunk_counts()
    ref = O.init(_op(sp))
    for t in range(nsteps):
        ref, rst = O.step(ref)
        assert stats[t].sums == rst.sums and stats[t].vmax2_bits == rst.vmax2_bits, t
    assert np.array_equal(fX, ref.X) and np.array_equal(fV, ref.V)
    assert sum(counts) >= spread.num_chunks * (1 if mode == "run" else 1)


def test_dynamic_slowed_position_takes_fewer_chunks():
    """Two positions on one GPU, position 1 spinning 2 ms per chunk task: the
    dynamic schedule moves work to position 0; the static one splits evenly.
    Results identical in both cases."""
    n, nsteps = (66, 40, 64), 4
    sp = P.SomierParams(n=n, seed=8)
    out = {}
    for sched in (P.SCHED_STATIC, P.SCHED_DYNAMIC):
        spread = P.Spread([0, 1], 1, n[0] - 2, chunk=4, sched=sched)
        with P.SomierStream(spread, sp, buffers=2, cuda_devices=[0, 0]) as s:
            s.set_delay(1, 2_000_000)
            X0, V0 = s.generate()
            X, V, XN = _pinned(X0.shape), _pinned(V0.shape), _pinned(X0.shape)
            X[...] = X0
            V[...] = V0
            st = s.run(X, V, XN, nsteps)
            out[sched] = (X.copy(), V.copy(), st[-1].sums, s.chunk_counts())
    xs, vs, ss, cs = out[P.SCHED_STATIC]
    xd, vd, sd, cd = out[P.SCHED_DYNAMIC]
    assert np.array_equal(xs, xd) and np.array_equal(vs, vd) and ss == sd
    nch = P.Spread([0, 1], 1, n[0] - 2, chunk=4).num_chunks
    assert cs == [nsteps * ((nch + 1) // 2), nsteps * (nch // 2)]
    assert sum(cd) == nsteps * nch and cd[1] < cd[0], cd


@pytest.mark.parametrize("chunk", [1, 7, 1000])
def test_dynamic_generic_loops(chunk):
    n = 20011
    A = np.random.default_rng(chunk).normal(size=n)
    dyn = P.Spread([0, 1, 2], 1, n - 2, chunk=chunk, sched=P.SCHED_DYNAMIC)
    # list ids 1, 2 do not exist on a one-GPU box: the generic loops bind list ids
    # directly, so only a one-position dynamic list runs here
    one = P.Spread([0], 1, n - 2, chunk=chunk, sched=P.SCHED_DYNAMIC)
    B = one.stencil3(A)
    assert np.array_equal(B[1:-1], O.stencil3(A)[1:-1])
    v, S, cnt = one.reduce(A)
    ref = O.reduce_exact(A, 1, n - 2, "sum", 60)
    assert S == ref[1] and v == ref[0] and cnt == n - 2
    assert dyn.dynamic and dyn.num_chunks == -(-(n - 2) // chunk)


def test_dynamic_resident_is_not_supported():
    sp = P.SomierParams(n=(10, 10, 10))
    with pytest.raises(P.SpreadError):
        P.Somier(P.Spread([0], 1, 8, chunk=2, sched=P.SCHED_DYNAMIC), sp)
