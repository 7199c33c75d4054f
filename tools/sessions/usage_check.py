import numpy as np
import paper_conf_ipps_torresft22_b200 as P
params = P.SomierParams(n=(64, 64, 64), seed=42)
with P.Somier(P.Spread([0], 1, 62), params) as s:
    s.step(10); st = s.stats(); X, V = s.read()
with P.SomierStream(P.Spread([0], 1, 62, chunk=16), params, buffers=2) as h:
    X2, V2 = h.generate()
    XN, VN = np.empty_like(X2), np.empty_like(V2)
    stats = h.run_blocked(X2, V2, XN, VN, nsteps=10, steps_per_trip=4)
# 3 trips -> odd -> state in (XN, VN)
assert np.array_equal(XN, X) and np.array_equal(VN, V) and stats[-1].sums == st.sums
total, S, count = P.Spread([0], 0, X[0].size, chunk=1 << 12).reduce(X[0].ravel(), "sum", 60)
assert S == st.sums[0], (S, st.sums[0])
print("usage ok", total / X[0].size, st.centre[0])
