"""Small end-to-end run of every step kernel for compute-sanitizer (tools/gpu_sanitize.sh).

Covers: the register SELL kernel, the TMA kernel on layout v0, the compact
encoding, the value-indexed kernel (16-, 8- and 31-warp tiles: the hot kernel
and its single-dictionary shape), the SMEM-resident kernel, the batched
value-indexed kernel (B = 2 and B = 8 on 15-warp tiles) and the GPU
enumerator.  (Not the in-process peer-memory rank group: its ranks' step
kernels wait on each other's flag barriers, and the sanitizer serialises
kernels, so they would wait out the barrier time-out.)
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import paper_conf_ipps_maggionibl13_b200 as cme  # noqa: E402
import workloads as W  # noqa: E402

KNOBS = [
    ("register", {"CME_TMA": "0", "CME_RESIDENT": "0"}),
    ("tma-v0", {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_COMPACT": "0"}),
    ("compact", {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_VI": "0"}),
    ("vi16", {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_VI": "1", "CME_VI2": "0", "CME_TMA_WARPS": "16"}),
    ("vi8", {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_VI": "1", "CME_VI2": "0", "CME_TMA_WARPS": "8"}),
    ("vi31", {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_VI": "1", "CME_VI2": "0", "CME_TMA_WARPS": "31"}),
    # tile-record kernel (sell_vi2_kernel, the cfg4 hot kernel): 30- and 16-warp
    # shapes, packed-word entries, and a capped grid that wraps the ring
    ("vi2-30", {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_VI": "1", "CME_VI2_WARPS": "30"}),
    ("vi2-16", {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_VI": "1", "CME_VI2_WARPS": "16"}),
    ("vi2-words", {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_VI": "1", "CME_VI2_WORDS": "1"}),
    ("vi2-grid2", {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_VI": "1", "CME_VI2_GRID": "2"}),
    # x window in shared memory (sell_vi2_kernel XWM 1 / 2): mirrored ring and
    # wrap mode, capped grid so each CTA's ring wraps
    ("xw-mirror", {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_XW": "1", "CME_XW_MODE": "1", "CME_VI2_GRID": "3"}),
    ("xw-wrap", {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_XW": "1", "CME_XW_MODE": "2", "CME_VI2_GRID": "3"}),
    ("resident", {"CME_TMA": "-1", "CME_RESIDENT": "1"}),
]
ALL_KEYS = sorted({k for _, kn in KNOBS for k in kn} | {"CME_TMA_WARPS", "CME_VI2_WARPS", "CME_XW", "CME_VI2B"})


def set_knobs(kn):
    for k in ALL_KEYS:
        os.environ.pop(k, None)
    os.environ.update(kn)


for label, knobs in KNOBS:
    set_knobs(knobs)
    for net, order in ((W.toggle_switch(30), cme.CME_ORDER_RCM), (W.schnakenberg(40), cme.CME_ORDER_NONE)):
        m = cme.Matrix.from_network(net).reorder(order).pack()
        m.set_opts(omega=0.9, check_every=7)
        p, st, it = m.solve(tol=1e-9, max_iter=300)
        y = m.spmv(W.random_start(m.n, 1))
        pt, terms = m.transient(0.05)
        f = m.info()
        print(label, net.name, "kernel", f.kernel, "compact", f.compact, "records", f.records, "warps", f.tma_warps, st, it,
              float(p.sum()), terms, flush=True)
        m.close()

# batches: the batched tile records (B = 2 default, B = 4 forced) and the
# batched value-indexed kernel (B = 8 on 15-warp tiles)
states, r, c, v = cme.cme_network_enumerate(W.toggle_switch(20))
for B, warps, extra in ((2, None, {}), (8, "15", {}), (4, None, {"CME_VI2B": "1"})):
    set_knobs({"CME_TMA": "1", "CME_RESIDENT": "-1"} | ({"CME_TMA_WARPS": warps} if warps else {}) | extra)
    vs = np.stack([v * (1.0 + 0.1 * b) for b in range(B)])
    m = cme.Matrix(len(states), r, c, vs).reorder(cme.CME_ORDER_RCM).pack()
    m.set_opts(omega=0.9, check_every=10)
    p, st, it = m.solve(tol=1e-9, max_iter=200)
    f = m.info()
    print("batch", B, "kernel", f.kernel, "compact", f.compact, "warps", f.tma_warps, st, it, flush=True)
    m.close()

# GPU state enumerator
for net in (W.toggle_switch(25), W.brusselator(30)):
    states, r, c, v = cme.cme_network_enumerate_gpu(net)
    print("gpu enumerate", net.name, len(states), len(r), flush=True)
print("sanitize case done")
