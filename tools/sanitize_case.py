"""Small end-to-end run of every step kernel for compute-sanitizer (tools/gpu_sanitize.sh)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import paper_conf_ipps_maggionibl13_b200 as cme  # noqa: E402
import workloads as W  # noqa: E402

for knobs in ({"CME_TMA": "0", "CME_RESIDENT": "0"}, {"CME_TMA": "1", "CME_RESIDENT": "0"},
              {"CME_TMA": "1", "CME_TMA_WARPS": "8", "CME_RESIDENT": "0"}, {"CME_TMA": "-1", "CME_RESIDENT": "1"}):
    os.environ.update(knobs)
    for net, order in ((W.toggle_switch(30), cme.CME_ORDER_RCM), (W.schnakenberg(40), cme.CME_ORDER_NONE)):
        m = cme.Matrix.from_network(net).reorder(order).pack()
        m.set_opts(omega=0.9, check_every=7)
        p, st, it = m.solve(tol=1e-9, max_iter=300)
        y = m.spmv(W.random_start(m.n, 1))
        pt, terms = m.transient(0.05)
        print(knobs, net.name, m.info().kernel, st, it, float(p.sum()), terms, flush=True)
        m.close()
    states, r, c, v = cme.cme_network_enumerate(W.toggle_switch(20))
    vs = np.stack([v * f for f in (1.0, 1.5)])
    os.environ["CME_RESIDENT"] = "-1"   # batches have no resident kernel
    m = cme.Matrix(len(states), r, c, vs).reorder(cme.CME_ORDER_RCM).pack()
    m.set_opts(omega=0.9, check_every=10)
    p, st, it = m.solve(tol=1e-9, max_iter=200)
    print(knobs, "batch2", m.info().kernel, st, it, flush=True)
    m.close()
# GPU state enumerator
for net in (W.toggle_switch(25), W.brusselator(30)):
    states, r, c, v = cme.cme_network_enumerate_gpu(net)
    print("gpu enumerate", net.name, len(states), len(r), flush=True)
print("sanitize case done")
