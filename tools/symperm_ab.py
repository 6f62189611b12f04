#!/usr/bin/env python3
"""Dev A/B: the 256-row local rearrangement (R13) as a row map inside the pack
(rows stay in RCM order, slots permuted) vs the same rearrangement folded into
the ordering (a symmetric permutation: slot = row, window 1)."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_maggionibl13_b200 as cme  # noqa: E402
import workloads as W  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "cfg4_toggle_20m"
net = W.config_network(name) if not name.startswith("toggle:") else W.toggle_switch(int(name.split(":")[1]))
states, r, c, v = cme.cme_network_enumerate(net)
n = len(states)
h = cme.Matrix(n, r, c, v).reorder(cme.CME_ORDER_RCM)
h.pack(cme.CME_FMT_DIAG_SELL, 256, cme.CME_BAND_AUTO, cme.CME_DEVICE_HOST_ONLY)
P = h.packed()
perm = h.permutation()
row_of = P["row_of"][:n]
composed = perm[row_of].astype(np.int32)
assert np.array_equal(np.sort(composed), np.arange(n))
h.close()


def timeit(m, label, blocks=10):
    f = m.info()
    st = torch.cuda.Stream()
    m.set_opts(omega=0.9, check_every=100, stream=st.cuda_stream)
    cme.cme_solver_load(m.h, n, None)
    cme.cme_solver_run(m.h, 3)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    cme.cme_solver_run(m.h, blocks)
    e1.record(st)
    torch.cuda.synchronize()
    t = e0.elapsed_time(e1) * 1e-3 / (blocks * 100)
    print(f"[{label}] {name} kernel={f.kernel} compact={f.compact} n_ell={f.n_ell} bytes_fmt={f.bytes_fmt} "
          f"t/iter={t * 1e6:.1f}us GFLOPS={2 * f.nnz / t / 1e9:.1f} fmt={f.bytes_fmt / t / 1e9:.0f}GB/s", flush=True)
    return m


for rep in range(2):
    a = cme.Matrix(n, r, c, v).reorder(cme.CME_ORDER_RCM).pack(cme.CME_FMT_DIAG_SELL, 256)
    timeit(a, "rowmap w256")
    pa, _, _ = a.solve(tol=1e-12)
    a.close()
    b = cme.Matrix(n, r, c, v).set_permutation(composed).pack(cme.CME_FMT_DIAG_SELL, 1)
    timeit(b, "symmetric w1")
    pb, _, _ = b.solve(tol=1e-12)
    b.close()
    print("L1(a-b)", float(np.abs(pa - pb).sum()), flush=True)
