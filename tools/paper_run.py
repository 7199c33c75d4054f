#!/usr/bin/env python3
"""The paper's experiment shape on one B200 (Table I):
Somier 1200^3, fp64, 31 time steps, state in HOST memory streamed through the
GPU every step. The paper's whole-program wall times (Table I,
PAPER.md:669-672) were 1058.9 s on 1 V100 and 502.0 s on 4 V100.

  python tools/paper_run.py [n] [steps] [chunk] [buffers] [run|step]

mode run (default): somier_stream_run, steps chained by per-chunk events (the
paper's future-work `depend`); step: somier_stream_step, a barrier per step
(the paper's taskgroup); run2: somier_stream_run2, two steps per host round
trip (12 host grids -- the paper's 154.5 GiB at 1200^3; refused if the host
has not that much memory available); blockedS (e.g. blocked8):
somier_stream_run_blocked with S steps per round trip (12 host grids).
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_torresft22_b200 as P  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1200
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 31
chunk = int(sys.argv[3]) if len(sys.argv) > 3 else 64
buffers = int(sys.argv[4]) if len(sys.argv) > 4 else 3
mode = sys.argv[5] if len(sys.argv) > 5 else "run"
ngrids = 12 if (mode == "run2" or mode.startswith("blocked")) else 9
need = ngrids * n ** 3 * 8
avail = 0
with open("/proc/meminfo") as f:
    for line in f:
        if line.startswith("MemAvailable:"):
            avail = int(line.split()[1]) * 1024
if avail < need * 1.1 + (16 << 30):
    print(json.dumps({"n": n, "mode": mode, "skipped": "host memory: need %.1f GiB pinned, %.1f GiB available" % (
        need / 2 ** 30, avail / 2 ** 30)}))
    sys.exit(0)
t_all = time.perf_counter()
params = P.SomierParams(n=(n, n, n), seed=42)
st = P.SomierStream(P.Spread([0], 1, n - 2, chunk=chunk), params, buffers=buffers)
t0 = time.perf_counter()
grids = [torch.empty((n, n, n), dtype=torch.float64, pin_memory=True) for _ in range(ngrids)]
t_pin = time.perf_counter() - t0
X, V, XN = [g.data_ptr() for g in grids[0:3]], [g.data_ptr() for g in grids[3:6]], [g.data_ptr() for g in grids[6:9]]
t0 = time.perf_counter()
st.generate_ptrs(X + V)
t_gen = time.perf_counter() - t0
per = []
t0 = time.perf_counter()
if mode == "run":
    stats = st.run_ptrs(X, V, XN, steps)[-1]
    per = [(time.perf_counter() - t0) / steps]
elif mode == "run2":
    VN = [g.data_ptr() for g in grids[9:12]]
    stats = st.run2_ptrs(X, V, XN, VN, steps)[-1]
    per = [(time.perf_counter() - t0) / steps]
elif mode.startswith("blocked"):
    VN = [g.data_ptr() for g in grids[9:12]]
    stats = st.run_blocked_ptrs(X, V, XN, VN, steps, int(mode[7:]))[-1]
    per = [(time.perf_counter() - t0) / steps]
else:
    for _ in range(steps):
        a = time.perf_counter()
        stats = st.step_ptrs(X, V, XN)
        per.append(time.perf_counter() - a)
        X, XN = XN, X
t_steps = time.perf_counter() - t0
tr = st.traffic()
if mode == "run2":  # bytes of one two-step launch, per step
    t2 = st.traffic2()
    tr = {"h2d_bytes": t2["h2d_bytes"] / 2, "d2h_bytes": t2["d2h_bytes"] / 2}
elif mode.startswith("blocked"):  # bytes of one trip, per step (full trips)
    S = int(mode[7:])
    t2 = st.traffic_blocked(S)
    tr = {"h2d_bytes": t2["h2d_bytes"] / S, "d2h_bytes": t2["d2h_bytes"] / S}
out = {"n": n, "steps": steps, "chunk": chunk, "buffers": buffers, "mode": mode,
       "host_state_gib": ngrids * n ** 3 * 8 / 2 ** 30,
       "pin_s": t_pin, "generate_s": t_gen, "steps_s": t_steps, "s_per_step": t_steps / steps,
       "per_step_min_max": [min(per), max(per)], "node_updates_per_s": (n - 2) ** 3 * steps / t_steps,
       "h2d_gb_per_step": tr["h2d_bytes"] / 1e9, "d2h_gb_per_step": tr["d2h_bytes"] / 1e9,
       "pcie_gbs": (tr["h2d_bytes"] + tr["d2h_bytes"]) / (t_steps / steps) / 1e9,
       "whole_program_s": time.perf_counter() - t_all, "centre": stats.centre, "vmax": stats.vmax,
       "paper_table1_s": {"1xV100 target spread": 1058.932, "4xV100 target spread": 502.019}}
print(json.dumps(out))
