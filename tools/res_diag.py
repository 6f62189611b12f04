"""Diagnostic: resident kernel vs register kernel vs oracle on a config-5 matrix."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import workloads as W
import oracle
import paper_conf_ipps_maggionibl13_b200 as cme

n = int(sys.argv[1]) if len(sys.argv) > 1 else 20000
width = int(sys.argv[2]) if len(sys.argv) > 2 else 16
r, c, v = W.banded_markov(n, 10, width, True, seed=5)
A = oracle.ingest(n, r, c, v)
for iters in (95, 1000, 5000):
    ref = oracle.jacobi_solve(A, omega=0.8, tol=0.0, check_every=10, max_iter=iters, stag_tol=0.0)
    for knob in ("0", "1"):
        os.environ["CME_RESIDENT"] = knob
        m = cme.Matrix(n, r, c, v).pack()
        m.set_opts(omega=0.8, check_every=10, stag_tol=0.0)
        p, st, it = m.solve(tol=0.0, max_iter=iters)
        rep = m.report()
        print(f"iters={iters} resident={knob} kernel={m.info().kernel} grid={m.info().grid} st={st} it={it} "
              f"L1={np.abs(p - ref.p).sum():.3e} delta={rep.delta:.3e} mass={rep.mass:.17g}", flush=True)
        m.close()
ref = oracle.jacobi_solve(A, omega=0.8, tol=1e-12, check_every=10, max_iter=100000, stag_tol=0.0)
print("oracle converge", ref.status, ref.iters, flush=True)
for knob in ("0", "1"):
    os.environ["CME_RESIDENT"] = knob
    m = cme.Matrix(n, r, c, v).pack()
    m.set_opts(omega=0.8, check_every=10, stag_tol=0.0)
    p, st, it = m.solve(tol=1e-12, max_iter=100000)
    rep = m.report()
    print(f"converge resident={knob} st={st} it={it} delta={rep.delta:.3e} L1={np.abs(p - ref.p).sum():.3e}", flush=True)
