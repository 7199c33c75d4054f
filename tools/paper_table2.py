#!/usr/bin/env python3
"""The paper's Table I / II comparison on one B200, in the
host-streamed mode: the grid lives in host memory and is mapped through the
GPU every step. Variants: One Buffer (1 device slot: H2D, kernel, D2H
serialised per chunk), double buffering (2 and 3 slots: the
copies of neighbouring chunks overlap the kernel).
Prints one JSON line per variant.

  python tools/paper_table2.py [n] [steps] [chunk]
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ipps_torresft22_b200 as P  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 10
chunk = int(sys.argv[3]) if len(sys.argv) > 3 else 32
params = P.SomierParams(n=(n, n, n), seed=42)
grids = [torch.empty((n, n, n), dtype=torch.float64, pin_memory=True) for _ in range(9)]
for buffers, name in ((1, "One Buffer (serialised)"), (2, "Double buffering, 2 slots"), (3, "Double buffering, 3 slots")):
    st = P.SomierStream(P.Spread([0], 1, n - 2, chunk=chunk), params, buffers=buffers)
    X, V, XN = [g.data_ptr() for g in grids[0:3]], [g.data_ptr() for g in grids[3:6]], \
        [g.data_ptr() for g in grids[6:9]]
    st.generate_ptrs(X + V)
    st.step_ptrs(X, V, XN)
    X, XN = XN, X
    t0 = time.perf_counter()
    for _ in range(steps):
        stats = st.step_ptrs(X, V, XN)
        X, XN = XN, X
    dt = time.perf_counter() - t0
    tr = st.traffic()
    st.close()
    print(json.dumps({"variant": name, "buffers": buffers, "n": n, "chunk": chunk, "steps": steps,
                      "s_per_step": dt / steps, "node_updates_per_s": (n - 2) ** 3 * steps / dt,
                      "pcie_gbs": (tr["h2d_bytes"] + tr["d2h_bytes"]) * steps / dt / 1e9, "vmax": stats.vmax}),
          flush=True)
