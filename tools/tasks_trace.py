#!/usr/bin/env python3
"""Trace of the chunk-level depend chain (SpreadTasks): enter A, B, C -> B =
S(A) -> C = S(B) -> reduce(C) -> exit C over 8 chunks (seven of 2^20 doubles,
the last of 100 x 2^20) of pinned arrays on devices(0..P-1) mapped to cuda:0;
prints one JSON line per chunk task (ms since tracing started) and a summary:
how many chunks' loops started before the LAST map(to) finished (a taskgroup
after the enter data would make that 0). The host-to-device copies of all
chunks share the copy engine, so equal chunks finish their copies together;
the big last chunk shows the chunk-level overlap.)"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_torresft22_b200 as P  # noqa: E402

sizes = [1 << 20] * 7 + [100 << 20]
n = sum(sizes) + 2
P_ = int(sys.argv[1]) if len(sys.argv) > 1 else 2
A = torch.empty(n, dtype=torch.float64, pin_memory=True).numpy()
A[:] = np.random.default_rng(1).normal(size=n)
Z = torch.zeros(n, dtype=torch.float64, pin_memory=True).numpy()
C = torch.zeros(n, dtype=torch.float64, pin_memory=True).numpy()
spread = P.Spread.with_sizes(list(range(P_)), 1, n - 2, sizes)
with P.SpreadTasks(spread, cuda_devices=[0] * P_) as q:
    q.set_trace(True)
    a = q.enter(A, lo_halo=1, hi_halo=1)
    b = q.enter(Z, lo_halo=1, hi_halo=1)
    c = q.enter(C)
    q.stencil3(a, b)
    q.stencil3(b, c)
    r = q.reduce_sum(c)
    q.exit(c, C)
    tr = q.trace()
    q.taskwait()
for rec in tr:
    print(json.dumps({"chunk": rec[0], "task": rec[1], "start_ms": round(rec[2], 4), "end_ms": round(rec[3], 4)}))
last_enter = max(e for _, k, _, e in tr if k == "enter")
first_loop = {}
for ch, k, s, e in tr:
    if k == "stencil3":
        first_loop[ch] = min(first_loop.get(ch, 1e30), s)
print(json.dumps({"summary": {"last_map_to_end_ms": last_enter, "loops_started_before_it": sum(
    1 for s in first_loop.values() if s < last_enter), "chunks": len(first_loop),
    "reduce_value": r.value, "end_ms": max(e for _, _, _, e in tr)}}))
