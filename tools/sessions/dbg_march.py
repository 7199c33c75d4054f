import paper_conf_ipps_torresft22_b200 as P
sp = P.SomierParams(n=(16,16,16), seed=1, kernel=P.K1_MARCH)
s = P.Somier(P.Spread([0],1,14), sp)
s.step(1)
print(s.stats())
