#!/usr/bin/env python3
"""Region-timed vs per-launch-bracketed K1_TB2 launches in one process (512^3):
does the timed region lose time between launches? Prints ms per launch."""
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch

import paper_conf_ipps_torresft22_b200 as P

n = int(sys.argv[1]) if len(sys.argv) > 1 else 512
s = P.Somier(P.Spread([0], 1, n - 2), P.SomierParams(n=[n, n, n], seed=42, kernel=P.K1_TB2))
st = torch.cuda.Stream()
s.set_stream(0, st.cuda_stream)
s.step(6)
s.sync()
L = 25
for rep in range(3):
    for mode in ("region", "bracketed", "region_nosleep"):
        if mode == "region":
            time.sleep(0.5)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        if mode.startswith("region"):
            e0.record(st)
            s.step(2 * L)
            e1.record(st)
            s.sync()
            print(rep, mode, "%.4f" % (e0.elapsed_time(e1) / L), flush=True)
        else:
            ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(L)]
            e0.record(st)
            for a, b in ev:
                a.record(st)
                s.step(2)
                b.record(st)
            e1.record(st)
            s.sync()
            d = [a.elapsed_time(b) for a, b in ev]
            print(rep, mode, "mean %.4f median %.4f first %.4f whole %.4f" % (
                statistics.mean(d), statistics.median(d), d[0], e0.elapsed_time(e1) / L), flush=True)
