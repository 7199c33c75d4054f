"""The single-process multi-device path on one GPU: list positions mapped to
the same CUDA device (somier_init_on) keep separate streams, so neighbouring
chunks on different positions exchange halos with the cross-device protocol
-- in-kernel stores into the neighbour's halo slot, release-stored completion
flags, cuStreamWaitValue64 before the next step -- exactly as between GPUs.
Results must be bit-identical to the oracle for every list, order and chunk."""
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


@pytest.mark.parametrize("devices,chunk", [([0, 1], 0), ([0, 1, 2, 3], 0), ([3, 1, 0, 2], 3), ([5, 7], 2),
                                           ([0, 1, 2], 1)])
@pytest.mark.parametrize("kernel", [P.K1_MARCH, P.K1_MARCH2, P.K1_DIRECT, P.K1_TB2])
@pytest.mark.parametrize("exchange", [P.EXCHANGE_FUSED, P.EXCHANGE_COPY])
def test_logical_devices_bit_identical(devices, chunk, kernel, exchange):
    n, steps = (22, 19, 45), 17
    sp = P.SomierParams(n=n, seed=11, kernel=kernel, exchange=exchange)
    spread = P.Spread(devices, 1, n[0] - 2, chunk=chunk)
    with P.Somier(spread, sp, cuda_devices=[0] * len(devices)) as s:
        s.step(5)
        s.step(1)
        s.step(steps - 6)
        st = s.stats()
        X, V = s.read()
    ref, rst = O.run(O.init(O.Params(n=n, seed=11)), steps)
    assert np.array_equal(X, ref.X) and np.array_equal(V, ref.V)
    assert st.sums == rst.sums and st.vmax2_bits == rst.vmax2_bits and st.centre == rst.centre


def test_logical_devices_load_and_continue():
    n = (14, 12, 33)
    sp = P.SomierParams(n=n, seed=2)
    with P.Somier(P.Spread([0, 1, 2], 1, n[0] - 2, chunk=2), sp, cuda_devices=[0, 0, 0]) as s:
        s.step(4)
        X, V = s.read()
        s.load(X, V)
        s.step(6)
        X2, V2 = s.read()
    ref, _ = O.run(O.init(O.Params(n=n, seed=2)), 10)
    assert np.array_equal(X2, ref.X) and np.array_equal(V2, ref.V)


@pytest.mark.parametrize("devices,sizes", [([0, 1], [3, 17]), ([0, 1, 2], [1, 8, 2, 5, 1, 3]), ([2, 0], [19, 1]),
                                           ([0], [4, 4, 12])])
@pytest.mark.parametrize("kernel", [P.K1_MARCH2, P.K1_DIRECT])
def test_irregular_spread_bit_identical(devices, sizes, kernel):
    """Irregular static schedule (spread_create_sizes): any chunk
    table gives the oracle's result bit for bit."""
    n, steps = (22, 19, 45), 13
    sp = P.SomierParams(n=n, seed=5, kernel=kernel)
    spread = P.Spread.with_sizes(devices, 1, n[0] - 2, sizes)
    with P.Somier(spread, sp, cuda_devices=[0] * len(devices)) as s:
        s.step(steps)
        st = s.stats()
        X, V = s.read()
    ref, rst = O.run(O.init(O.Params(n=n, seed=5)), steps)
    assert np.array_equal(X, ref.X) and np.array_equal(V, ref.V)
    assert st.sums == rst.sums and st.vmax2_bits == rst.vmax2_bits


def test_weighted_spread_bit_identical():
    n = (40, 16, 33)
    sp = P.SomierParams(n=n, seed=8)
    with P.Somier(P.Spread.weighted([0, 1, 2], 1, n[0] - 2, [1.0, 3.0, 0.5]), sp, cuda_devices=[0, 0, 0]) as s:
        s.step(9)
        X, V = s.read()
    ref, _ = O.run(O.init(O.Params(n=n, seed=8)), 9)
    assert np.array_equal(X, ref.X) and np.array_equal(V, ref.V)


@pytest.mark.parametrize("devices,sizes", [([0, 1], [3, 17]), ([0, 1, 2], [2, 8, 2, 5, 3]), ([2, 0], [18, 2]),
                                           ([0], [4, 4, 12]), ([0, 1], [2, 2, 2, 2, 2, 2, 2, 2, 2, 2])])
def test_tb2_deep_halo_spreads_bit_identical(devices, sizes):
    """K1_TB2 on several chunks: two X halo planes and one V halo plane per face,
    stored by the neighbour's kernel (cross-stream flags between list
    positions, stream order within one); chunks of two planes (both halo planes
    from one neighbour); pairs and single steps, on either parity."""
    n = (22, 19, 45)
    sp = P.SomierParams(n=n, seed=7, kernel=P.K1_TB2)
    spread = P.Spread.with_sizes(devices, 1, n[0] - 2, sizes)
    with P.Somier(spread, sp, cuda_devices=[0] * len(devices)) as s:
        assert s.kernel_in_use == P.K1_TB2
        done = 0
        for k in (4, 1, 3, 2, 5):
            s.step(k)
            done += k
            st = s.stats()
            ref, rst = O.run(O.init(O.Params(n=n, seed=7)), done)
            assert st.sums == rst.sums and st.vmax2_bits == rst.vmax2_bits, (k, done)
        X, V = s.read()
    assert np.array_equal(X, ref.X) and np.array_equal(V, ref.V)


def test_tb2_one_plane_chunk_falls_back():
    """A chunk of one plane among several cannot feed a neighbour's two halo
    planes: K1_TB2 resolves to K1_MARCH2 (still bit-identical)."""
    n = (14, 12, 33)
    sp = P.SomierParams(n=n, seed=2, kernel=P.K1_TB2)
    with P.Somier(P.Spread.with_sizes([0, 1], 1, n[0] - 2, [1, 11]), sp, cuda_devices=[0, 0]) as s:
        assert s.kernel_in_use == P.K1_MARCH2
        s.step(5)
        X, V = s.read()
    ref, _ = O.run(O.init(O.Params(n=n, seed=2)), 5)
    assert np.array_equal(X, ref.X) and np.array_equal(V, ref.V)


@pytest.mark.parametrize("chunk", [0, 2, 3])
def test_tb2_load_and_continue(chunk):
    """somier_load fills the deep halo planes (X two, V one per face) too."""
    n = (14, 12, 33)
    sp = P.SomierParams(n=n, seed=2, kernel=P.K1_TB2)
    with P.Somier(P.Spread([0, 1, 2], 1, n[0] - 2, chunk=chunk), sp, cuda_devices=[0, 0, 0]) as s:
        s.step(3)
        X, V = s.read()
        s.load(X, V)
        s.step(7)
        X2, V2 = s.read()
        st = s.stats()
    ref, rst = O.run(O.init(O.Params(n=n, seed=2)), 10)
    assert np.array_equal(X2, ref.X) and np.array_equal(V2, ref.V)
    assert st.sums == rst.sums and st.vmax2_bits == rst.vmax2_bits


@pytest.mark.parametrize("kernel", [P.K1_MARCH2, P.K1_TB2, P.K1_DIRECT])
@pytest.mark.parametrize("chunk", [2, 3, 7])
def test_nccl_exchange_self_send_bitwise(kernel, chunk):
    """SOMIER_EXCHANGE_NCCL on one GPU: every chunk boundary goes through
    ncclSend / ncclRecv (one list position = one rank, so the boundaries are
    self send/recv on its stream) -- the route's buffers, plane offsets and
    message order, bitwise against the oracle."""
    n, steps = (22, 19, 45), 13
    sp = P.SomierParams(n=n, seed=11, kernel=kernel, exchange=P.EXCHANGE_NCCL)
    with P.Somier(P.Spread([0], 1, n[0] - 2, chunk=chunk), sp) as s:
        s.step(5)
        s.step(steps - 5)
        st = s.stats()
        X, V = s.read()
    ref, rst = O.run(O.init(O.Params(n=n, seed=11)), steps)
    assert np.array_equal(X, ref.X) and np.array_equal(V, ref.V)
    assert st.sums == rst.sums and st.vmax2_bits == rst.vmax2_bits


def test_nccl_exchange_needs_distinct_gpus():
    """NCCL places one rank per GPU: two list positions on one device are refused."""
    sp = P.SomierParams(n=(12, 10, 10), exchange=P.EXCHANGE_NCCL)
    with pytest.raises(P.SpreadError) as e:
        P.Somier(P.Spread([0, 1], 1, 10), sp, cuda_devices=[0, 0])
    assert e.value.status == P._native.ENOTSUP
    import ctypes
    uid = ctypes.create_string_buffer(128)
    P._native.check(P._native.lib().somier_nccl_unique_id(uid), "somier_nccl_unique_id")
    assert any(uid.raw)
