"""spread_reduce (the reduction clause of the paper's future work, PAPER.md:330,
773): every chunk reduced on its device, partials combined; bit-identical to
the definition (oracle.reduce_exact) for every schedule."""
import math

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


def _data(n, seed, scale=30):
    """Values over 12 decades (|a| < 2^24, inside the sum's domain for scale <= 69),
    signed zeros, and two exact ties at the given scale."""
    rng = np.random.default_rng(seed)
    a = np.clip(rng.standard_normal(n), -4, 4) * 10.0 ** rng.integers(-6, 6, n)
    a[::97] = 0.0
    a[1::101] = -0.0
    a[5] = 0.5 * 2.0 ** -scale  # a tie: rounds to even (0)
    a[6] = 1.5 * 2.0 ** -scale  # tie: rounds to 2
    return a


@pytest.mark.parametrize("chunk", [0, 1, 7, 1000, 10 ** 6])
@pytest.mark.parametrize("op", ["sum", "min", "max"])
def test_reduce_equals_definition_any_chunking(op, chunk):
    n = 12345
    a = _data(n, 3)
    v, S, cnt = P.Spread([0], 2, n - 5, chunk=chunk).reduce(a, op, 30)
    wv, wS = O.reduce_exact(a, 2, n - 5, op, 30)
    assert cnt == n - 5
    assert S == wS
    assert v == wv and math.copysign(1.0, v) == math.copysign(1.0, wv)


@pytest.mark.parametrize("sizes", [[1, 2, 3, 10], [10, 1, 5], [16]])
def test_reduce_irregular_and_scales(sizes):
    for scale in (-10, 0, 30, 36):
        a = _data(16, 5, scale)
        v, S, _ = P.Spread.with_sizes([0], 0, 16, sizes).reduce(a, "sum", scale)
        assert (v, S) == O.reduce_exact(a, 0, 16, "sum", scale)


def test_reduce_large_exact_and_order_independent():
    """10^7 elements: the exact sum does not depend on the chunking (and equals
    the definition); the naive float sum of the same data does."""
    n = 10 ** 7
    rng = np.random.default_rng(11)
    a = rng.uniform(-1e3, 1e3, n)
    res = {P.Spread([0], 0, n, chunk=c).reduce(a, "sum", 40)[:2] for c in (0, 123457, 10 ** 6)}
    assert len(res) == 1
    (v, S), = res
    # the definition, vectorised: a * 2^40 is exact and below 2^50, rint rounds half to even
    assert S == sum(np.rint(a * 2.0 ** 40).astype(np.int64).tolist())


def test_reduce_nan_empty_and_domain():
    a = np.array([1.0, np.nan, -3.0, 2.0])
    assert math.isnan(P.Spread([0], 0, 4, chunk=2).reduce(a, "max")[0])
    assert math.isnan(P.Spread([0], 0, 4, chunk=2).reduce(a, "min")[0])
    assert P.Spread([0], 2, 2, chunk=1).reduce(a, "min")[0] == -3.0
    assert P.Spread([0], 2, 0).reduce(a, "max")[0] == -math.inf
    assert P.Spread([0], 2, 0).reduce(a, "sum")[:2] == (0.0, 0)
    with pytest.raises(P.SpreadError):
        P.Spread([0], 0, 4).reduce(a, "sum")  # NaN is outside the sum's domain
    with pytest.raises(P.SpreadError):
        P.Spread([0], 0, 2).reduce(np.array([1.0, 2.0 ** 34]), "sum", 60)  # 2^94
    with pytest.raises(P.SpreadError):
        P.Spread([0], 0, 5).reduce(a, "sum")  # range outside the array


def test_reduce_reproduces_somier_centre_sums():
    """The Somier "centers" reduction through the generic clause:
    the x coordinates of a state summed at scale 2^60 over a spread give the
    exact sums somier_stats reports."""
    sp = P.SomierParams(n=(12, 10, 14), seed=2)
    with P.Somier(P.Spread([0], 1, 10), sp) as s:
        s.step(3)
        X, _ = s.read()
        st = s.stats()
    for c in range(3):
        flat = np.ascontiguousarray(X[c]).ravel()
        _, S, _ = P.Spread([0], 0, flat.size, chunk=97).reduce(flat, "sum", 60)
        assert S == st.sums[c]
