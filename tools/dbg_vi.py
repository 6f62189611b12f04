import os, numpy as np, sys
sys.path.insert(0, os.getcwd())
import paper_conf_ipps_maggionibl13_b200 as cme, workloads as W
os.environ["CME_TMA"]="1"; os.environ["CME_RESIDENT"]="0"
states, r, c, v = cme.cme_network_enumerate(W.toggle_switch(90))
res={}
for enc, env in (("v0", {"CME_COMPACT": "0"}), ("vi", {"CME_COMPACT": "1", "CME_VI": "1"}), ("cpt", {"CME_COMPACT": "1", "CME_VI": "0"})):
    os.environ.update(env)
    m = cme.Matrix(len(states), r, c, v).reorder(cme.CME_ORDER_RCM).pack()
    f=m.info(); print(enc, f.compact, f.tma_warps, f.tma_stages, f.grid)
    m.set_opts(omega=0.9, check_every=50, stag_tol=0.0)
    res[enc]={}
    for it in (1,2,3,49,50,51,52,100,300):
        p, st, k = m.solve(tol=0.0, max_iter=it)
        res[enc][it]=p
for it in res["v0"]:
    a,b,c2=res["v0"][it],res["vi"][it],res["cpt"][it]
    print(it, "vi==v0", a.tobytes()==b.tobytes(), "maxrel", np.max(np.abs(a-b)/a), "cpt-v0", np.max(np.abs(a-c2)/a))
