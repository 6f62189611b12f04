#!/usr/bin/env python3
"""Format / ordering ablation on B200: the analogues of the
paper's Table II (ELL vs ELL+DIA), Table III (ELL / sliced ELL / warp-grained
ELL) and the reordering study of P:L225 (random / global / local), measured as
fp64 Jacobi-step GFLOPS with the library's kernels.

    python tools/ablation.py [--configs cfg3a_schnakenberg_2m,cfg4_toggle_20m] [--out FILE]

Every variant is one cme_pack of the same ingested matrix; timing = CUDA events
over 10 check blocks (1000 iterations) after 3 warm-up blocks.
"""
import argparse
import json
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
ap.add_argument("--configs", default="cfg3a_schnakenberg_2m,cfg3b_brusselator_2m,cfg4_toggle_20m,toggle1_table1")
ap.add_argument("--blocks", type=int, default=10)
ap.add_argument("--out", default=None)
a = ap.parse_args()

PEAK = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))).get("hbm_gbs", 6543.4) \
    if os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6543.4
F = cme
VARIANTS = [  # name, order, fmt, window, band
    ("ELL", "natural", F.CME_FMT_ELL, 1, F.CME_BAND_NEVER),
    ("ELL+DIA", "natural", F.CME_FMT_ELL, 1, F.CME_BAND_AUTO),
    ("SlicedELL256", "natural", F.CME_FMT_SELL256, 1, F.CME_BAND_NEVER),
    ("WarpedELL", "natural", F.CME_FMT_DIAG_SELL, 1, F.CME_BAND_NEVER),
    ("WarpedELL+local", "natural", F.CME_FMT_DIAG_SELL, 256, F.CME_BAND_NEVER),
    ("WarpedELL+local+DIA", "natural", F.CME_FMT_DIAG_SELL, 256, F.CME_BAND_AUTO),
    ("WarpedELL+global", "natural", F.CME_FMT_DIAG_SELL, 1 << 30, F.CME_BAND_NEVER),
    ("WarpedELL+local+DIA/RCM", "rcm", F.CME_FMT_DIAG_SELL, 256, F.CME_BAND_AUTO),
    ("WarpedELL+local/random", "random", F.CME_FMT_DIAG_SELL, 256, F.CME_BAND_NEVER),
    ("CSR", "natural", F.CME_FMT_CSR, 1, F.CME_BAND_NEVER),
]


def network(name):
    if name == "toggle1_table1":   # Table I toggle-switch-1 (N = 400)
        return W.toggle_switch(400), 0.9
    return W.config_network(name), W.CONFIGS[name]["omega"]


rows = []
for cfg in a.configs.split(","):
    net, omega = network(cfg)
    s, r, c, v = cme.cme_network_enumerate(net)
    n = len(s)
    rng_perm = np.random.default_rng(1).permutation(n).astype(np.int32)
    for name, order, fmt, window, band in VARIANTS:
        m = cme.Matrix(n, r, c, v)
        if order == "rcm":
            m.reorder(cme.CME_ORDER_RCM)
        elif order == "random":
            m.set_permutation(rng_perm)
        t0 = time.time()
        m.pack(fmt, window, band)
        f = m.info()
        st = torch.cuda.Stream()
        m.set_opts(omega=omega, check_every=100, stream=st.cuda_stream)
        cme.cme_solver_load(m.h, n, None)
        cme.cme_solver_run(m.h, 3)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        cme.cme_solver_run(m.h, a.blocks)
        e1.record(st)
        torch.cuda.synchronize()
        ti = e0.elapsed_time(e1) * 1e-3 / (100 * a.blocks)
        row = dict(config=cfg, variant=name, order=order, n=f.n, nnz=f.nnz, band_on=bool(f.band_on),
                   ell_efficiency=round(f.ell_efficiency, 4), kernel=int(f.kernel), encoding=int(f.compact),
                   records=int(f.records), xwin_kb=int(f.xwin_kb),
                   packed_mib=round(f.packed_bytes / 2 ** 20, 2), bytes_fmt=f.bytes_fmt,
                   us_per_iter=round(ti * 1e6, 2), gflops=round(2 * f.nnz / ti / 1e9, 1),
                   alg_gbs=round(f.bytes_alg / ti / 1e9, 1), pct_peak=round(100 * f.bytes_alg / ti / 1e9 / PEAK, 1),
                   fmt_gbs=round(f.bytes_fmt / ti / 1e9, 1))
        rows.append(row)
        print(json.dumps(row), flush=True)
        m.close()
if a.out:
    with open(a.out, "w") as fh:
        json.dump(rows, fh, indent=1)
