#!/usr/bin/env python3
"""Dev tool: time the fused step under different kernel knobs on one workload.

    python tools/kbench.py [--config cfg4_toggle_20m] [--blocks 10] VAR=VAL,VAR=VAL ...

Each positional argument is one variant: comma-separated environment
assignments (CME_TMA, CME_TMA_STAGES, CME_TMA_CTAS, ...) applied before
re-packing.  Prints per-iteration time, GFLOPS and GB/s (B_alg and B_fmt).
"""
import argparse
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import workloads as W  # noqa: E402
import paper_conf_ipps_maggionibl13_b200 as cme  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="cfg4_toggle_20m")
ap.add_argument("--order", default=None)
ap.add_argument("--window", type=int, default=256)
ap.add_argument("--band", type=int, default=0)
ap.add_argument("--fmt", type=int, default=0)
ap.add_argument("--blocks", type=int, default=10)
ap.add_argument("--C", type=int, default=100)
ap.add_argument("--batch", type=int, default=1)
ap.add_argument("variants", nargs="*", default=[""])
a = ap.parse_args()

if a.config.startswith("banded"):
    _, n, mu, w, irr = a.config.split(":")
    r, c, v = W.banded_markov(int(n), int(mu), int(w), irr == "1", 1)
    n = int(n)
    omega = 1.0
    order = a.order or "none"
elif a.config.startswith("toggle:"):   # toggle switch with buffer N (Table I toggle-switch-1: N = 400)
    s, r, c, v = cme.cme_network_enumerate(W.toggle_switch(int(a.config.split(":")[1])))
    n = len(s)
    omega = 0.9
    order = a.order or "rcm"
else:
    t = time.time()
    if a.batch > 1:
        vs = []
        for net in W.sweep_networks(a.config, a.batch):
            s, r, c, v = cme.cme_network_enumerate(net)
            vs.append(v)
        v = np.stack(vs)
    else:
        s, r, c, v = cme.cme_network_enumerate(W.config_network(a.config))
    n = len(s)
    omega = W.CONFIGS[a.config]["omega"]
    order = a.order or ("rcm" if "toggle" in a.config else "none")
    print(f"enumerated n={n} in {time.time() - t:.1f}s", flush=True)
m = cme.Matrix(n, r, c, v)
m.reorder({"none": 0, "dfs": 1, "rcm": 2}[order])
del r, c, v
peak = 6543.4
for var in a.variants:
    env = dict(kv.split("=") for kv in var.split(",") if kv)
    old = {k: os.environ.get(k) for k in env}
    os.environ.update(env)
    m.pack(a.fmt, a.window, a.band)
    for k, val in old.items():
        if val is None:
            os.environ.pop(k)
        else:
            os.environ[k] = val
    f = m.info()
    st = torch.cuda.Stream()
    m.set_opts(omega=omega, check_every=a.C, stream=st.cuda_stream)
    cme.cme_solver_load(m.h, n * a.batch, None)
    cme.cme_solver_run(m.h, 3)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    cme.cme_solver_run(m.h, a.blocks)
    e1.record(st)
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    it = a.blocks * a.C
    ti = ms * 1e-3 / it
    print(f"[{var or 'default'}] {a.config} B={a.batch} kernel={f.kernel} order={order} n={f.n} nnz={f.nnz} "
          f"band={f.band_on} rec={f.records} wf={f.wf_steps}/{f.wf_lag} warps={f.tma_warps} st={f.tma_stages} t/iter={ti * 1e6:.1f}us GFLOPS={2 * f.nnz * a.batch / ti / 1e9:.1f} "
          f"alg={f.bytes_alg / ti / 1e9:.0f}GB/s ({100 * f.bytes_alg / ti / 1e9 / peak:.1f}%) "
          f"fmt={f.bytes_fmt / ti / 1e9:.0f}GB/s", flush=True)
