#!/usr/bin/env python3
"""Host C++ of libcme under AddressSanitizer + UndefinedBehaviorSanitizer (no GPU).

    python tools/asan_host.py            # builds libcme_asan.so, re-runs itself under LD_PRELOAD=libasan

Builds the library with the host code instrumented (`build.py --sanitize`,
-fsanitize=address,undefined, no recovery from UB) and drives every host path
of the C ABI that runs without a device: network enumeration, COO/CSR/batch
ingest incl. duplicates and the error paths, DFS/RCM/caller permutations,
the period test, packing every format/window/band with CME_DEVICE_HOST_ONLY
(layout v0, compact and value-indexed encodings, tile records), the export
views, the partition/halo plan at 2-4 ranks.  Any report aborts the process
(exit != 0).  The log is committed as profiles/sanitizer/round2_host_asan_ubsan.txt.
"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_ipps_maggionibl13_b200", "libcme_asan.so")


def exercise():
    sys.path.insert(0, ROOT)
    import numpy as np
    import paper_conf_ipps_maggionibl13_b200 as cme
    import workloads as W
    n_calls = 0
    nets = [W.toggle_switch(30), W.brusselator(25), W.schnakenberg(20), W.birth_death(100), W.schlogl(150),
            W.cyclic3(4)]
    for net in nets:
        states, r, c, v = cme.cme_network_enumerate(net)
        n = len(states)
        for order in (cme.CME_ORDER_NONE, cme.CME_ORDER_DFS, cme.CME_ORDER_RCM):
            for fmt, window, band in ((cme.CME_FMT_DIAG_SELL, 256, cme.CME_BAND_AUTO),
                                      (cme.CME_FMT_DIAG_SELL, 1, cme.CME_BAND_ALWAYS),
                                      (cme.CME_FMT_ELL, 1, cme.CME_BAND_NEVER),
                                      (cme.CME_FMT_SELL256, 256, cme.CME_BAND_AUTO),
                                      (cme.CME_FMT_CSR, 1, cme.CME_BAND_NEVER)):
                m = cme.Matrix(n, r, c, v)
                m.reorder(order)
                m.pack(fmt, window, band, cme.CME_DEVICE_HOST_ONLY)
                m.info()
                m.packed()
                if fmt == cme.CME_FMT_DIAG_SELL:
                    try:
                        m.compact()
                    except cme.CmeError:
                        pass
                m.permutation()
                cme.cme_period(m.h)
                m.close()
                n_calls += 1
        # caller permutation, batch ingest, partition plans
        m = cme.Matrix(n, r, c, v)
        m.set_permutation(np.random.default_rng(1).permutation(n).astype(np.int32))
        m.pack(cme.CME_FMT_DIAG_SELL, 256, cme.CME_BAND_AUTO, cme.CME_DEVICE_HOST_ONLY)
        m.close()
        vb = np.stack([v, 2.0 * v])
        h = cme.cme_matrix_create_coo_batch(n, r, c, vb)
        cme.cme_reorder(h, cme.CME_ORDER_RCM)
        cme.cme_pack(h, cme.CME_FMT_DIAG_SELL, 256, cme.CME_BAND_AUTO, cme.CME_DEVICE_HOST_ONLY)
        cme.cme_matrix_destroy(h)
        for P in (2, 3, 4):
            for rank in range(P):
                m = cme.Matrix(n, r, c, v).reorder(cme.CME_ORDER_RCM)
                m.pack(cme.CME_FMT_DIAG_SELL, 64, cme.CME_BAND_AUTO, cme.CME_DEVICE_HOST_ONLY)
                cme.cme_matrix_plan_partition(m.h, P, rank)
                cme.cme_export_halo(m.h)
                m.packed()
                m.close()
                n_calls += 1
    # error paths: negative rate, NaN, zero outflow, out-of-range index, duplicates, bad call order
    r = np.array([1, 0, 1, 1], np.int32)
    c = np.array([0, 1, 0, 0], np.int32)
    for rate in ([1.0, 2.0, -1.0, 0.5], [1.0, float("nan"), 1.0, 1.0], [1.0, 2.0, 3.0, 4.0]):
        try:
            cme.Matrix(2, r, c, np.array(rate)).close()
        except cme.CmeError:
            pass
    for bad in ((np.array([5], np.int32), np.array([0], np.int32)), (np.array([0], np.int32), np.array([0], np.int32))):
        try:
            cme.Matrix(2, bad[0], bad[1], np.array([1.0])).close()
        except cme.CmeError:
            pass
    m = cme.Matrix(2, np.array([0, 1], np.int32), np.array([1, 0], np.int32), np.array([1.0, 2.0]))
    try:
        m.solve(tol=1e-12, max_iter=10)   # before pack: BAD_STATE
    except cme.CmeError:
        pass
    m.close()
    print(f"asan/ubsan host exercise: {n_calls} pack/plan calls on {len(nets)} networks + error paths: clean", flush=True)


def main():
    if os.environ.get("CME_ASAN_CHILD") == "1":
        exercise()
        return 0
    sys.path.insert(0, os.path.join(ROOT, "paper_conf_ipps_maggionibl13_b200"))
    import build as B
    B.build(out=LIB, sanitize=True)
    asan = subprocess.run(["gcc", "-print-file-name=libasan.so"], capture_output=True, text=True).stdout.strip()
    ubsan = subprocess.run(["gcc", "-print-file-name=libubsan.so"], capture_output=True, text=True).stdout.strip()
    env = dict(os.environ, CME_ASAN_CHILD="1", CME_LIBRARY=LIB, LD_PRELOAD=f"{asan}:{ubsan}",
               ASAN_OPTIONS="detect_leaks=0:abort_on_error=1:halt_on_error=1",
               UBSAN_OPTIONS="print_stacktrace=1:halt_on_error=1")
    return subprocess.call([sys.executable, os.path.abspath(__file__)], env=env)


if __name__ == "__main__":
    sys.exit(main())
