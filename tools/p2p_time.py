"""Time free-running check blocks of a row-sharded solve over the peer-memory
group (virtual ranks = host threads on one GPU) vs the single-GPU handle."""
import os
import sys
import threading
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_ipps_maggionibl13_b200 as cme  # noqa: E402
import workloads as W  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "cfg2_toggle_100k"
nranks = int(sys.argv[2]) if len(sys.argv) > 2 else 2
blocks = int(sys.argv[3]) if len(sys.argv) > 3 else 5
s, r, c, v = cme.cme_network_enumerate(W.config_network(cfg))
n = len(s)
m = cme.Matrix(n, r, c, v).reorder(2).pack()
m.set_opts(omega=0.9)
cme.cme_solver_load(m.h, n, None)
cme.cme_solver_run(m.h, 2)
torch.cuda.synchronize()
t = time.perf_counter()
cme.cme_solver_run(m.h, blocks)
torch.cuda.synchronize()
single = (time.perf_counter() - t) / (blocks * 100)
m.close()
comms = cme.cme_comm_init_local([0] * nranks)
times = [0.0] * nranks


def worker(k):
    mm = cme.Matrix(n, r, c, v).reorder(2)
    mm.pack(device=cme.CME_DEVICE_HOST_ONLY)
    cme.cme_matrix_distribute(mm.h, comms[k])
    mm.set_opts(omega=0.9)
    cme.cme_solver_load(mm.h, n, None)
    cme.cme_solver_run(mm.h, 2)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    cme.cme_solver_run(mm.h, blocks)
    torch.cuda.synchronize()
    times[k] = (time.perf_counter() - t0) / (blocks * 100)
    p, st, it = mm.solve(tol=0.0, max_iter=100)   # a barrier time-out would surface here
    if st != "NOT_CONVERGED":
        print(f"rank {k}: status {st} after the timed blocks", flush=True)
    mm.close()


th = [threading.Thread(target=worker, args=(k,)) for k in range(nranks)]
[t.start() for t in th]
[t.join() for t in th]
print(f"{cfg} n={n}: single {single * 1e6:.1f} us/iter; {nranks} virtual ranks on one GPU: "
      f"{max(times) * 1e6:.1f} us/iter (max over ranks)")
