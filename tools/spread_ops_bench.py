#!/usr/bin/env python3
"""Throughput of the spread runtime's generic loops on one B200: the paper's
Listing 3 stencil (spread_stencil3: map(to: A[start-1:size+2]) -> kernel ->
map(from: B[start:size])) and the reduction clause (spread_reduce: map(to:
A[start:size]) -> on-device reduction), on PINNED host arrays, against the
measured host<->device copy rates -- both are bound by the host link, as
every `target spread` loop over host data is. One JSON line
per (op, chunk).

  python tools/spread_ops_bench.py [n_doubles]
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_torresft22_b200 as P  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 28  # 2 GiB of doubles
A = torch.empty(n, dtype=torch.float64, pin_memory=True)
B = torch.empty(n, dtype=torch.float64, pin_memory=True)
A.uniform_(-1.0, 1.0)
a, b = A.numpy(), B.numpy()

# measured pinned copy rates (one direction, and both at once)
d = torch.empty(n, dtype=torch.float64, device="cuda")
for name, fn in (("h2d", lambda: d.copy_(A, non_blocking=True)), ("d2h", lambda: B.copy_(d, non_blocking=True))):
    fn()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    fn()
    torch.cuda.synchronize()
    rate = n * 8 / (time.perf_counter() - t0) / 1e9
    print(json.dumps({"copy": name, "gbs": rate}), flush=True)
del d
torch.cuda.empty_cache()

for chunk in (1 << 22, 1 << 24, 1 << 26):
    sp = P.Spread([0], 1, n - 2, chunk=chunk)
    sp.stencil3(a, b)  # warm-up
    t0 = time.perf_counter()
    sp.stencil3(a, b)
    dt = time.perf_counter() - t0
    print(json.dumps({"op": "stencil3", "n": n, "chunk": chunk, "s": dt, "elements_per_s": (n - 2) / dt,
                      "host_link_gbs": 2 * (n - 2) * 8 / dt}), flush=True)
    sp = P.Spread([0], 0, n, chunk=chunk)
    for op in ("sum", "max"):
        sp.reduce(a, op, 40)
        t0 = time.perf_counter()
        v = sp.reduce(a, op, 40)
        dt = time.perf_counter() - t0
        print(json.dumps({"op": "reduce_" + op, "n": n, "chunk": chunk, "s": dt, "elements_per_s": n / dt,
                          "h2d_gbs": n * 8 / dt, "value": v[0]}), flush=True)
