#!/usr/bin/env python3
"""Small runs of every kernel path for compute-sanitizer (tests/test_gpu_sanitizer.py):
K1 direct / march / march2 over a multi-chunk spread (fused halo stores), the
host-streamed mode (one and two steps per round trip), K2 and K3, and K1_TB2 on a
single chunk."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import paper_conf_ipps_torresft22_b200 as P  # noqa: E402

n = (10, 19, 37)
for kern in (P.K1_DIRECT, P.K1_MARCH, P.K1_MARCH2):
    sp = P.SomierParams(n=n, seed=3, kernel=kern)
    with P.Somier(P.Spread([0], 1, n[0] - 2, chunk=3), sp) as s:
        s.step(3)
        s.stats()
        X, V = s.read()
        s.load(X, V)
        s.step(1)
        s.sync()
    with P.SomierStream(P.Spread([0], 1, n[0] - 2, chunk=4), sp, buffers=2) as st:
        X, V = st.generate()
        XN = np.zeros_like(X)
        st.step(X, V, XN)
# K1_TB2 (AUTO on a large single chunk): two steps per launch, shared-memory rings and
# the one-plane-ahead border springs; odd step counts take the one-step path too
for kern in (P.K1_TB2,):
    sp = P.SomierParams(n=n, seed=3, kernel=kern)
    with P.Somier(P.Spread([0], 1, n[0] - 2), sp) as s:
        assert s.kernel_in_use == P.K1_TB2
        s.step(5)
        s.stats()
        s.step(2)
        s.sync()
    # host-streamed, two steps per round trip (somier_stream_run2), odd count
    with P.SomierStream(P.Spread([0], 1, n[0] - 2, chunk=3), sp, buffers=2) as st:
        X, V = st.generate()
        st.run2(X, V, np.zeros_like(X), np.zeros_like(V), 3)
        st.run_blocked(X, V, np.zeros_like(X), np.zeros_like(V), 7, 5)
# the reduction clause over a multi-chunk spread
a = np.linspace(-3.0, 5.0, 1001)
for op in ("sum", "min", "max"):
    P.Spread([0], 1, 999, chunk=37).reduce(a, op, 40)
print("sanitize case ok")
