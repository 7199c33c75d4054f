#!/usr/bin/env python3
"""Small runs of every kernel path for compute-sanitizer (tests/test_gpu_sanitizer.py):
K1 direct / march / march2 over a multi-chunk spread (fused halo stores), the
host-streamed mode (one and two steps per round trip, dynamic schedule), K2 and
K3, K1_TB2 on a single chunk and across positions (every step's stats), the
copy and NCCL exchange routes, and the task queue's chained constructs."""
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
    # every step's stats from the history ring (both steps of a launch)
    with P.Somier(P.Spread([0, 1], 1, n[0] - 2, chunk=4), sp, cuda_devices=[0, 0]) as s:
        s.step(6)
        s.stats_history(1, 6)
# the exchange routes across list positions: copies after the kernel, and NCCL (self send/recv)
for ex in (P.EXCHANGE_COPY, P.EXCHANGE_NCCL):
    sp = P.SomierParams(n=n, seed=3, kernel=P.K1_MARCH2, exchange=ex)
    devs = [0, 1] if ex == P.EXCHANGE_COPY else [0]
    with P.Somier(P.Spread(devs, 1, n[0] - 2, chunk=3), sp, cuda_devices=[0] * len(devs)) as s:
        s.step(3)
        s.sync()
# dynamic schedule in the host-streamed mode
sp = P.SomierParams(n=n, seed=3)
with P.SomierStream(P.Spread([0, 1], 1, n[0] - 2, chunk=2, sched=P.SCHED_DYNAMIC), sp, buffers=2,
                    cuda_devices=[0, 0]) as st:
    X, V = st.generate()
    st.run(X, V, np.zeros_like(X), 3)
# the reduction clause over a multi-chunk spread
a = np.linspace(-3.0, 5.0, 1001)
for op in ("sum", "min", "max"):
    P.Spread([0], 1, 999, chunk=37).reduce(a, op, 40)
# chunk-level depend between constructs (task queue, halo refresh by peer copies)
with P.SpreadTasks(P.Spread([0, 1], 1, 999, chunk=97), cuda_devices=[0, 0]) as q:
    ta = q.enter(a, lo_halo=1, hi_halo=1)
    tb = q.enter(np.zeros_like(a), lo_halo=1, hi_halo=1)
    tc = q.enter(np.zeros_like(a))
    q.stencil3(ta, tb)
    q.stencil3(tb, tc)
    q.reduce_sum(tc)
    out = np.zeros_like(a)
    q.exit(tc, out)
    q.taskwait()
print("sanitize case ok")
