#!/usr/bin/env python3
"""Host-streamed Somier, steps per host round trip swept on one B200: the state
(12 pinned host grids) is generated once, then for every (chunk, s) the same
nsteps are run through somier_stream_run (s = 1, one step per trip, V in
place) or somier_stream_run_blocked (s >= 2) and timed by wall clock (every
copy, kernel and the per-trip stats read-back inside). Prints one JSON line
per configuration.

  python tools/stream_blocked_sweep.py n nsteps chunk:s[:buffers] [...]   (buffers default 3)
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_torresft22_b200 as P  # noqa: E402

n = int(sys.argv[1])
nsteps = int(sys.argv[2])
cfgs = [tuple(int(v) for v in (c + ":3").split(":")[:3]) for c in sys.argv[3:]]
need = 12 * n ** 3 * 8
with open("/proc/meminfo") as f:
    avail = next(int(line.split()[1]) * 1024 for line in f if line.startswith("MemAvailable:"))
if avail < need * 1.1 + (16 << 30):
    print(json.dumps({"n": n, "skipped": "host memory: need %.1f GiB, %.1f GiB available" % (need / 2 ** 30,
                                                                                            avail / 2 ** 30)}))
    sys.exit(0)
params = P.SomierParams(n=(n, n, n), seed=42)
t0 = time.perf_counter()
grids = [torch.empty((n, n, n), dtype=torch.float64, pin_memory=True) for _ in range(12)]
pin_s = time.perf_counter() - t0
ptr = [g.data_ptr() for g in grids]
X, V, XN, VN = ptr[0:3], ptr[3:6], ptr[6:9], ptr[9:12]
ref = None
for chunk, s, buffers in cfgs:
    st = P.SomierStream(P.Spread([0], 1, n - 2, chunk=chunk), params, buffers=buffers)
    st.generate_ptrs(X + V)
    t0 = time.perf_counter()
    if s == 1:
        stats = st.run_ptrs(X, V, XN, nsteps)[-1]
        tr = st.traffic()
        per_step = tr["h2d_bytes"] + tr["d2h_bytes"]
    else:
        stats = st.run_blocked_ptrs(X, V, XN, VN, nsteps, s)[-1]
        tr = st.traffic_blocked(s)
        per_step = (tr["h2d_bytes"] + tr["d2h_bytes"]) / s
    wall = time.perf_counter() - t0
    st.close()
    key = (stats.sums, stats.vmax2_bits)
    ref = ref or key
    print(json.dumps({"n": n, "nsteps": nsteps, "chunk": chunk, "steps_per_trip": s, "buffers": buffers, "wall_s": wall,
                      "node_updates_per_s": (n - 2) ** 3 * nsteps / wall,
                      "host_bytes_per_node_update": per_step / (n - 2) ** 3,
                      "pcie_gbs": per_step * nsteps / wall / 1e9, "pin_s": pin_s,
                      "same_final_stats_as_first_config": key == ref, "vmax": stats.vmax}), flush=True)
