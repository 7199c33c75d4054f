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


def test_no_barrier_between_constructs():
    """No taskgroup between the constructs, shown deterministically: chunk 5's
    stream is held (it waits on a host word) before its map(to); every other
    chunk's whole chain -- map(to) of A and B, both stencil loops, map(from)
    of C -- completes while chunk 5 has not even started (under the paper's
    taskgroup no loop could run before every map(to) finished). Only the two
    neighbours of chunk 5 could need its data: their halo element comes from
    chunk 5's enter data, so they are held too -- and released with it."""
    import time

    n = 1 << 16
    A = torch.empty(n, dtype=torch.float64, pin_memory=True).numpy()
    A[:] = np.random.default_rng(1).normal(size=n)
    Z = torch.zeros(n, dtype=torch.float64, pin_memory=True).numpy()
    C = torch.full((n,), np.nan, dtype=torch.float64, pin_memory=True).numpy()
    spread = P.Spread([0, 1], 1, n - 2, chunk=(n - 2 + 7) // 8)
    ch = spread.chunks()
    with P.SpreadTasks(spread, cuda_devices=[0, 0]) as q:
        q.hold(5)
        a = q.enter(A, lo_halo=1, hi_halo=1)
        b = q.enter(Z, lo_halo=1, hi_halo=1)
        c = q.enter(Z)
        q.stencil3(a, b)
        q.stencil3(b, c)
        q.exit(c, C)
        # chunks far from 5 finish while chunk 5 waits (their results land in C)
        far = [k for k in range(8) if abs(k - 5) > 2]
        deadline = time.time() + 30
        done = lambda: all(not np.isnan(C[ch[k].start:ch[k].start + ch[k].size]).any() for k in far)  # noqa: E731
        while not done() and time.time() < deadline:
            time.sleep(0.01)
        assert done(), "chunks away from the held one did not complete"
        held = C[ch[5].start:ch[5].start + ch[5].size]
        assert np.isnan(held).all(), "the held chunk ran"
        q.release()
        q.taskwait()
    B = np.zeros(n)
    B[1:-1] = O.stencil3(A)[1:-1]
    Cref = np.zeros(n)
    Cref[1:-1] = O.stencil3(B)[1:-1]
    assert np.array_equal(C[1:-1], Cref[1:-1])


def test_trace_records_follow_the_dependencies():
    """The trace API: one record per chunk task, each chunk's loop after its own
    map(to) of A and its map(from) after its loop (the chunk-level order; how
    the copies of different chunks interleave is the copy engines' business)."""
    sizes = [1 << 18] * 7 + [1 << 20]
    n = sum(sizes) + 2
    A = torch.empty(n, dtype=torch.float64, pin_memory=True).numpy()
    A[:] = np.random.default_rng(1).normal(size=n)
    Bh = torch.zeros(n, dtype=torch.float64, pin_memory=True).numpy()
    spread = P.Spread.with_sizes([0], 1, n - 2, sizes)
    with P.SpreadTasks(spread) as q:
        q.set_trace(True)
        b = q.enter(None, n=n)  # map(alloc: B[...]): B is only written
        a = q.enter(A, lo_halo=1, hi_halo=1)
        q.stencil3(a, b)
        q.exit(b, Bh)
        tr = q.trace()
        q.taskwait()
    rec = {}
    for c, k, s0, e0 in tr:
        rec.setdefault((c, k), []).append((s0, e0))
    for c in range(8):
        assert len(rec[(c, "enter")]) == 2 and len(rec[(c, "stencil3")]) == 1 and len(rec[(c, "exit")]) == 1
        a_end = rec[(c, "enter")][1][1]
        loop = rec[(c, "stencil3")][0]
        assert loop[0] >= a_end and rec[(c, "exit")][0][0] >= loop[1]
    ref = O.stencil3(A)
    assert np.array_equal(Bh[1:-1], ref[1:-1])
