#!/usr/bin/env python3
"""Config 5 (BASELINE.json configs[4]): synthetic banded Markov generator sweep,
1M-100M rows, varying bandwidth and irregularity -> fused Jacobi step GB/s vs
the HBM roofline ("SpMV GB/s vs roofline surface").

    python tools/sweep_cfg5.py [--quick] [--out profiles/round1_cfg5_sweep]

Per point: the C generator (workloads.banded_markov_fast, identical to the
numpy definition), ingest + natural order + DIAG+SELL pack (auto band: the
j+-1 backbone always makes the band dense), then the library's free-running
check blocks timed with CUDA events on the solver's stream (3 warm-up blocks,
then `--blocks` blocks of C = 100 steps).  Every point also checks the
|d|-weighted mass invariant of one omega = 1 SpMV (sum |a_jj| y_j = sum
|a_jj| x_j), which holds at any size.  Bytes: B_alg = 12 nnz + 16 n
(SURVEY 8(d)); B_fmt = the layout's compulsory bytes (cme_info.bytes_fmt).
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

M = 1_000_000


def points(quick):
    if quick:
        return [(1 * M, 10, 1024, False), (4 * M, 10, 32, False), (4 * M, 10, 4 * M, False)]
    pts = [(n, 10, 1024, False) for n in (1 * M, 4 * M, 16 * M, 64 * M, 100 * M)]
    pts += [(16 * M, 10, w, False) for w in (32, 4096, 8192, 32768, 1 * M, 16 * M)]
    pts += [(16 * M, 10, 4096, True)]
    pts += [(16 * M, mu, 1024, irr) for mu in (5, 7, 15) for irr in (False, True)]
    pts += [(16 * M, 10, 1024, True), (64 * M, 10, 32768, True)]
    return pts


def peak_gbs():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6543.4, "fallback"


def run_point(n, mu, w, irr, blocks, C=100):
    t = time.time()
    r, c, v = W.banded_markov_fast(n, mu, w, irr, seed=1)
    t_gen = time.time() - t
    d = np.bincount(c, weights=v, minlength=n)          # |a_jj| = column sums (sanity check only)
    t = time.time()
    m = cme.Matrix(n, r, c, v)
    del r, c, v
    m.pack()
    t_pack = time.time() - t
    f = m.info()
    x = W.random_start(n, 7)
    m.set_opts(omega=1.0)
    y = m.spmv(x)
    inv = abs((d * y).sum() - (d * x).sum()) / (d * x).sum()
    st = torch.cuda.Stream()
    m.set_opts(omega=1.0, check_every=C, stream=st.cuda_stream)
    cme.cme_solver_load(m.h, n, None)
    cme.cme_solver_run(m.h, 3)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    cme.cme_solver_run(m.h, blocks)
    e1.record(st)
    torch.cuda.synchronize()
    ti = e0.elapsed_time(e1) * 1e-3 / (blocks * C)
    out = dict(n=n, mu=mu, width=w, irregular=irr, nnz=int(f.nnz), kernel=int(f.kernel), band_on=int(f.band_on),
               encoding=int(f.compact), records=int(f.records), xwin_kb=int(f.xwin_kb),
               us_per_iter=ti * 1e6, gflops=2 * f.nnz / ti / 1e9, alg_gbs=f.bytes_alg / ti / 1e9,
               fmt_gbs=f.bytes_fmt / ti / 1e9, bytes_alg=int(f.bytes_alg), bytes_fmt=int(f.bytes_fmt),
               mass_invariant_rel=float(inv), gen_s=round(t_gen, 2), ingest_pack_s=round(t_pack, 2))
    m.close()
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--blocks", type=int, default=10)
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "cfg5_sweep"))
    a = ap.parse_args()
    peak, src = peak_gbs()
    rows = []
    import psutil
    for p in points(a.quick):
        need = 60 * p[0] * p[1]          # ~60 B of host memory per generated entry (COO + ingest + pack)
        avail = psutil.virtual_memory().available
        if need > 0.7 * avail:
            print(json.dumps(dict(n=p[0], mu=p[1], width=p[2], irregular=p[3],
                                  skipped=f"needs ~{need / 1e9:.0f} GB host memory, {avail / 1e9:.0f} GB free")),
                  flush=True)
            continue
        o = run_point(*p, blocks=a.blocks)
        o["frac_alg"] = o["alg_gbs"] / peak
        o["frac_fmt"] = o["fmt_gbs"] / peak
        assert o["mass_invariant_rel"] <= 1e-12, o
        rows.append(o)
        print(json.dumps(o), flush=True)
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    with open(a.out + ".json", "w") as f:
        json.dump(dict(peak_gbs=peak, peak_source=src, points=rows), f, indent=1)
    kn = {0: "register", 1: "tma", 2: "csr"}
    enc = {0: " (v0)", 1: " (compact)", 2: " (value-indexed)"}
    with open(a.out + ".md", "w") as f:
        f.write(f"# Config 5 sweep: synthetic banded Markov generator, fused Jacobi step on one B200\n\n"
                f"Peak {peak:.1f} GB/s ({src}). `alg` = B_alg = 12 nnz + 16 n per iteration; `fmt` = the "
                f"packed layout's compulsory bytes (of the encoding the kernel streams). Natural order, DIAG+SELL, "
                f"auto band, omega = 1.\n\n"
                "| n | mu | width | irregular | nnz | kernel | us/iter | GFLOPS | alg GB/s | % peak (alg) | "
                "fmt GB/s | % peak (fmt) |\n|---|---|---|---|---|---|---|---|---|---|---|---|\n")
        for o in rows:
            f.write(f"| {o['n']:,} | {o['mu']} | {o['width']:,} | {int(o['irregular'])} | {o['nnz']:,} | "
                    f"{kn.get(o['kernel'], o['kernel'])}{enc.get(o.get('encoding', 0), '')}"
                    f"{' + records' if o.get('records') else ''}"
                    f"{(' + x window %d KB' % o['xwin_kb']) if o.get('xwin_kb') else ''} | "
                    f"{o['us_per_iter']:.1f} | {o['gflops']:.0f} | "
                    f"{o['alg_gbs']:.0f} | {100 * o['frac_alg']:.1f} | {o['fmt_gbs']:.0f} | "
                    f"{100 * o['frac_fmt']:.1f} |\n")


if __name__ == "__main__":
    main()
