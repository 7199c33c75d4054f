"""The paper's example loop (Listing 3/4) run by the spread runtime on the GPU:
bit-identical to the oracle's left-to-right B[i] = A[i-1] + A[i] + A[i+1]
for every chunking (the paper's N = 14 with chunk 4 and 2 included) and for
sub-ranges of the loop."""
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


@pytest.mark.parametrize("n,chunk", [(14, 4), (14, 2), (1000, 7), (100003, 0), (100003, 4096), (3, 1)])
def test_stencil3_equals_oracle(n, chunk):
    A = np.random.default_rng(n).normal(size=n)
    B = P.Spread([0], 1, n - 2, chunk=chunk).stencil3(A)
    ref = O.stencil3(A)
    assert np.array_equal(B, ref)


def test_stencil3_subrange_leaves_rest_untouched():
    A = np.arange(50, dtype=np.float64) ** 1.5
    B = np.full(50, -7.0)
    P.Spread([0], 10, 20, chunk=6).stencil3(A, B)
    ref = O.stencil3(A)
    assert np.array_equal(B[10:30], ref[10:30])
    assert (B[:10] == -7).all() and (B[30:] == -7).all()


@pytest.mark.parametrize("sizes", [[1, 5, 2, 4], [12], [3, 3, 1, 1, 1, 1, 1, 1]])
def test_stencil3_irregular_chunks(sizes):
    A = np.random.default_rng(len(sizes)).normal(size=14)
    B = P.Spread.with_sizes([0], 1, 12, sizes).stencil3(A)
    assert np.array_equal(B, O.stencil3(A))
