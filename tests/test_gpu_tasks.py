"""Chunk-level `depend` between spread constructs (SpreadTasks, include/spread.h;
PAPER.md:746-767, Listing 13): enter data -> stencil loop -> stencil loop ->
reduction -> exit data chained per chunk with no taskgroup in between. Results
must equal the oracle's sequential loops bit for bit on regular and irregular
chunk tables over several list positions (logical devices on one GPU, halo
copies between positions), and a trace must show a chunk's loop running before
the next chunk's map(to) has finished (no barrier between the constructs)."""
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


def _spread(devices, n, chunk=None, sizes=None):
    if sizes is not None:
        return P.Spread.with_sizes(devices, 1, n - 2, sizes)
    return P.Spread(devices, 1, n - 2, chunk=chunk)


@pytest.mark.parametrize("devices,n,chunk,sizes", [
    ([0], 14, 4, None), ([0, 1], 14, 2, None), ([2, 0, 1], 1003, 7, None), ([0, 1, 2, 3], 100003, 0, None),
    ([0, 1], 14, None, [1, 5, 2, 4]), ([1, 0, 2], 14, None, [3, 3, 1, 1, 1, 1, 1, 1]), ([0], 3, 1, None)])
def test_chain_equals_oracle(devices, n, chunk, sizes):
    rng = np.random.default_rng(n)
    A = rng.normal(size=n)
    B0 = np.full(n, 0.25)        # B's elements outside the loop (B[0], B[n-1]) enter from the host
    C0 = np.full(n, -1.5)
    spread = _spread(devices, n, chunk, sizes)
    with P.SpreadTasks(spread, cuda_devices=[0] * len(devices)) as q:
        a = q.enter(A, lo_halo=1, hi_halo=1)
        b = q.enter(B0, lo_halo=1, hi_halo=1)
        c = q.enter(C0)
        q.stencil3(a, b)          # B = stencil(A): depend(in: A[start-1:size+2]) depend(out: B[start:size])
        q.stencil3(b, c)          # C = stencil(B): B's halo comes from the neighbour chunks' B
        r = q.reduce_sum(c)       # reduction(+: sum C[range])
        Bh, Ch = np.full(n, np.nan), np.full(n, np.nan)
        q.exit(b, Bh)
        q.exit(c, Ch)
        q.taskwait()
    Bref = B0.copy()
    Bref[1:n - 1] = O.stencil3(A)[1:n - 1]
    Cref = C0.copy()
    Cref[1:n - 1] = O.stencil3(Bref)[1:n - 1]
    assert np.array_equal(Bh[1:n - 1], Bref[1:n - 1]) and np.isnan(Bh[0]) and np.isnan(Bh[n - 1])
    assert np.array_equal(Ch[1:n - 1], Cref[1:n - 1])
    ref = O.reduce_exact(Cref, 1, n - 2, "sum", 60)
    assert (r.sum_hi << 64) + r.sum_lo == ref[1] and r.value == ref[0] and r.count == n - 2


def test_war_rewrite_after_reads():
    """A data written again after other chunks read its halo: the rewrite waits
    for those reads (WAR), the second read sees the new values (RAW)."""
    n = 4001
    A = np.random.default_rng(3).normal(size=n)
    spread = P.Spread([0, 1, 2], 1, n - 2, chunk=97)
    with P.SpreadTasks(spread, cuda_devices=[0, 0, 0]) as q:
        a = q.enter(A, lo_halo=1, hi_halo=1)
        b = q.enter(np.zeros(n), lo_halo=1, hi_halo=1)
        q.stencil3(a, b)   # B1 = S(A)
        q.stencil3(b, a)   # A2 = S(B1): A rewritten while its chunks' halos were read above
        q.stencil3(a, b)   # B2 = S(A2)
        Bh = np.zeros(n)
        q.exit(b, Bh)
        q.taskwait()
    A1 = A.copy()
    B1 = np.zeros(n)
    B1[1:-1] = O.stencil3(A1)[1:-1]
    A2 = A1.copy()
    A2[1:-1] = O.stencil3(B1)[1:-1]
    B2 = B1.copy()
    B2[1:-1] = O.stencil3(A2)[1:-1]
    assert np.array_equal(Bh[1:-1], B2[1:-1])


def test_no_barrier_between_constructs_trace():
    """Pinned host arrays over 8 chunks whose last one is 100x larger: with
    chunk-level dependencies the stencil of the small chunks starts while the
    big chunk's map(to) is still running -- under the paper's taskgroup no loop
    could start before every map(to) of the enter data had finished."""
    small, big = 1 << 20, 100 << 20
    sizes = [small] * 7 + [big]
    n = sum(sizes) + 2
    A = torch.empty(n, dtype=torch.float64, pin_memory=True).numpy()
    A[:] = np.random.default_rng(1).normal(size=n)
    Bh = torch.zeros(n, dtype=torch.float64, pin_memory=True).numpy()
    spread = P.Spread.with_sizes([0], 1, n - 2, sizes)
    with P.SpreadTasks(spread) as q:
        q.set_trace(True)
        a = q.enter(A, lo_halo=1, hi_halo=1)
        b = q.enter(Bh, lo_halo=1, hi_halo=1)
        q.stencil3(a, b)
        q.exit(b, Bh)
        tr = q.trace()
        q.taskwait()
    enters = [(c, s, e) for c, k, s, e in tr if k == "enter"]
    loops = [(c, s, e) for c, k, s, e in tr if k == "stencil3"]
    assert len(enters) == 16 and len(loops) == 8
    last_enter_end = max(e for _, _, e in enters)
    assert min(s for _, s, _ in loops) < last_enter_end, (enters, loops)
    ref = O.stencil3(A)
    assert np.array_equal(Bh[1:-1], ref[1:-1])
