#!/usr/bin/env python3
"""Power split probe: board power / SM clock while running (a) a sustained
torch copy at full HBM bandwidth, (b) K1 at 512^3 back to back. Tells how
much of the 1 kW budget the memory side and the fp64 side of K1 take."""
import statistics
import subprocess
import sys
import time

sys.path.insert(0, ".")
import torch  # noqa: E402


def sample(fn, seconds=3.0):
    q = "power.draw,clocks.sm,clocks.mem"
    p = subprocess.Popen(["nvidia-smi", "-i", "0", "--query-gpu=" + q, "--format=csv,noheader,nounits", "-lms", "50"],
                         stdout=subprocess.PIPE, text=True)
    time.sleep(0.3)
    t0 = time.time()
    n = 0
    while time.time() - t0 < seconds:
        fn()
        n += 1
    torch.cuda.synchronize()
    p.terminate()
    out = p.communicate()[0].strip().splitlines()
    vals = [[float(x) for x in l.split(",")] for l in out[len(out) // 3:]]
    return {"power_w": statistics.median(v[0] for v in vals), "sm_mhz": statistics.median(v[1] for v in vals),
            "iters": n}


torch.cuda.set_device(0)
a = torch.empty(6 * (1 << 30) // 8, dtype=torch.float64, device="cuda").fill_(1.0)
b = torch.empty_like(a)
print("copy", sample(lambda: [b.copy_(a) for _ in range(10)]))
del a, b
torch.cuda.empty_cache()
import paper_conf_ipps_torresft22_b200 as P  # noqa: E402
for k in (P.K1_MARCH, P.K1_MARCH2):
    s = P.Somier(P.Spread([0], 1, 510), P.SomierParams(n=(512, 512, 512), kernel=k))
    r = sample(lambda: s.step(20))
    s.sync()
    print("k1", k, r)
    s.close()
x = torch.ones(1 << 20, dtype=torch.float64, device="cuda")
print("idle-ish", sample(lambda: time.sleep(0.05), 1.0))
