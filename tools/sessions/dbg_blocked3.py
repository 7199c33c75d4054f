import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_ipps_torresft22_b200 as P
exec(open(os.path.join(os.path.dirname(__file__), "dbg_blocked.py")).read().split("cases =")[0])
for n, chunk, s, nsteps, b in [((300, 512, 512), 300, 2, 2, 1), ((300, 512, 512), 64, 2, 2, 1), ((300, 512, 512), 64, 4, 4, 1)] * 4:
    ref = run(n, chunk, 1, 3, nsteps)
    got = run(n, chunk, s, b, nsteps)
    for name, g, r in (("X", got[0], ref[0]), ("V", got[1], ref[1])):
        bad = ~(g == r)
        planes = sorted(set(np.argwhere(bad)[:, 1].tolist()))
        print(n, chunk, s, nsteps, "buffers", b, os.environ.get("SOMIER_TB2_NSEG"), name, "bad", int(bad.sum()), "planes", planes[:12], len(planes), flush=True)
