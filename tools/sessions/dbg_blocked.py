import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_ipps_torresft22_b200 as P
def run(n, chunk, s, buffers, nsteps, pinned=True):
    sp = P.SomierParams(n=n, seed=42)
    st = P.SomierStream(P.Spread([0], 1, n[0]-2, chunk=chunk), sp, buffers=buffers)
    mk = (lambda: torch.empty((3,)+tuple(n), dtype=torch.float64, pin_memory=True).numpy()) if pinned else (lambda: np.zeros((3,)+tuple(n)))
    X, V, XN, VN = mk(), mk(), mk(), mk()
    X0, V0 = st.generate(); X[...] = X0; V[...] = V0; XN[...] = np.nan; VN[...] = np.nan
    if s == 1:
        stats = st.run(X, V, XN, nsteps); fX, fV = (X, V) if nsteps % 2 == 0 else (XN, V)
    else:
        stats = st.run_blocked(X, V, XN, VN, nsteps, s); nt = -(-nsteps // s); fX, fV = (X, V) if nt % 2 == 0 else (XN, VN)
    st.close()
    return fX.copy(), fV.copy(), stats[-1]
cases = [((512, 512, 512), 64, 8, 32), ((512, 256, 256), 64, 8, 32), ((300, 512, 512), 64, 8, 32)] if len(sys.argv) > 1 else [((40, 33, 70), 16, 8, 16), ((100, 64, 64), 32, 8, 16), ((200, 64, 64), 64, 8, 16), ((200, 128, 128), 64, 8, 32), ((300, 256, 256), 64, 8, 32)]
for n, chunk, s, nsteps in cases:
    ref = run(n, chunk, 1, 3, nsteps)
    for b in (1, 1, 2):
        for pinned in (True,):
            got = run(n, chunk, s, b, nsteps, pinned)
            okx = np.array_equal(got[0], ref[0]); okv = np.array_equal(got[1], ref[1])
            bad = np.argwhere(~(got[0] == ref[0]))
            print(n, chunk, s, nsteps, 'buffers', b, 'pinned', pinned, okx, okv, got[2].sums == ref[2].sums, bad[:3].tolist() if len(bad) else '', flush=True)
