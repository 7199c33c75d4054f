"""The optional all-cores oracle build (oracle/liboracle_omp.so: the same
somier_oracle.c compiled with -fopenmp, bench.py's second CPU-baseline line)
must be bit-identical to the sequential oracle: every node is computed by the
same expressions whichever thread runs it, and the centre sums are exact
("bitwise equal to the sequential run because nodes are
independent and stats are exact"). Also pins oracle_run_timed to oracle_run."""
import numpy as np
import pytest

import oracle as O


@pytest.mark.parametrize("n,steps", [((9, 7, 11), 12), ((34, 5, 17), 6), ((3, 3, 3), 4), ((12, 40, 9), 5)])
def test_omp_build_bit_identical(n, steps):
    s0 = O.init(O.Params(n=n, seed=13, mass=1.7, rest_len=0.9))
    ref, rst = O.run(s0, steps)
    seq, sst, sec, thr = O.run_timed(s0, steps)
    assert thr == 1 and sec >= 0.0
    assert np.array_equal(seq.X, ref.X) and np.array_equal(seq.V, ref.V) and sst == rst
    par, pst, psec, pthr = O.run_timed(s0, steps, omp=True)
    assert pthr >= 1 and psec >= 0.0
    assert np.array_equal(par.X, ref.X) and np.array_equal(par.V, ref.V) and pst == rst
