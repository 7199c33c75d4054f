#!/usr/bin/env python3
"""Diagnose the steady-state slowdown of K1: per-step CUDA-event times over a
long run next to nvidia-smi samples (clocks, power, temperatures, reasons)."""
import json
import subprocess
import sys
import time

sys.path.insert(0, ".")
import torch  # noqa: E402

import paper_conf_ipps_torresft22_b200 as P  # noqa: E402

steps = int(sys.argv[1]) if len(sys.argv) > 1 else 400
n = int(sys.argv[2]) if len(sys.argv) > 2 else 512
out = sys.argv[3] if len(sys.argv) > 3 else "gpurun_out/diag"
torch.cuda.set_device(0)
s = P.Somier(P.Spread([0], 1, n - 2), P.SomierParams(n=(n, n, n), seed=42))
st = torch.cuda.Stream()
s.set_stream(0, st.cuda_stream)
s.step(3)
s.sync()
q = ("timestamp,clocks.sm,clocks.mem,power.draw,temperature.gpu,temperature.memory,"
     "clocks_event_reasons.active,clocks_event_reasons.sw_power_cap,clocks_event_reasons.hw_slowdown,"
     "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown")
smi = subprocess.Popen(["nvidia-smi", "-i", "0", "--query-gpu=" + q, "--format=csv,noheader", "-lms", "20"],
                       stdout=open(out + "_smi.csv", "w"), stderr=subprocess.DEVNULL)
time.sleep(0.5)
ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
t0 = time.time()
for i in range(steps):
    ev[i][0].record(st)
    s.step(1)
    ev[i][1].record(st)
s.sync()
t1 = time.time()
time.sleep(0.5)
smi.terminate()
ms = [b.elapsed_time(e) for b, e in ev]
json.dump({"t0": t0, "t1": t1, "ms": ms}, open(out + "_steps.json", "w"))
for i in range(0, steps, max(1, steps // 20)):
    print(i, "%.3f" % ms[i])
print("mean first 20 %.3f last 20 %.3f" % (sum(ms[:20]) / 20, sum(ms[-20:]) / 20))
