#!/usr/bin/env python3
"""Proxy for the multi-GPU protocol cost on a one-GPU box: the N-way spread of
one grid over N list positions that all map to cuda:0 (somier_init_on), each
position with its own stream, chunk boundaries exchanged by the fused peer
stores + device flags exactly as between GPUs. Total node-updates/s for
N = 1, 2, 4, 8 on the same GPU: the drop from N = 1 is what the chunking,
deep-halo exchange and flag waits cost (the GPU's SMs are shared, so this is
not a scaling measurement). Host wall clock around step(K) + sync.

Usage: python tools/logical_scale.py [n] [steps] [exchange: fused|copy]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_ipps_torresft22_b200 as P  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 40
exchange = {"fused": P.EXCHANGE_FUSED, "copy": P.EXCHANGE_COPY}[sys.argv[3] if len(sys.argv) > 3 else "fused"]
torch.cuda.init()
res = {}
for rep in range(2):
    for L in (1, 2, 4, 8):
        sp = P.SomierParams(n=[n, n, n], seed=42, exchange=exchange)
        with P.Somier(P.Spread(list(range(L)), 1, n - 2), sp, cuda_devices=[0] * L) as s:
            s.step(6)
            s.sync()
            t0 = time.perf_counter()
            s.step(steps)
            s.sync()
            dt = time.perf_counter() - t0
            st = s.stats()
            v = (n - 2) ** 3 * steps / dt
            res.setdefault(L, []).append(v)
            print(json.dumps({"n": n, "positions": L, "exchange": sys.argv[3] if len(sys.argv) > 3 else "fused", "kernel": s.kernel_in_use, "launches_per_step": s.launches /
                              max(1, s.step_count), "node_updates_per_s": v, "ms_per_step": dt / steps * 1e3,
                              "centre0": st.centre[0], "vmax": st.vmax}), flush=True)
best1 = max(res[1])
print(json.dumps({"summary": {str(L): max(v) / best1 for L, v in res.items()}}))
