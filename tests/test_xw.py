"""GPU parity of the x-window step kernel (sell_vi2_kernel<..., XW = true>,
DESIGN.md sec. 5f): each CTA runs a contiguous range of tiles and reads the
iterate from a shared-memory ring that its producer warp streams with the tile
records.  Same arithmetic as the tile-record kernel (FMAs in t order, row sum
times inv_d), so the tolerances are those of tests/test_gpu_parity.py:
one Jacobi application <= 1e-13 componentwise, fixed-iteration landscapes
<= 1e-12 L1, converged landscapes <= 1e-10 L1 (eq. 8).

Capped grids (2-5 CTAs) make every CTA stream hundreds of tiles, so the x
ring wraps many times and the chunk-release rule (a chunk is overwritten only
after every tile that reads it has released its stage) is exercised.
"""
import numpy as np
import pytest

import workloads as W
from test_gpu_parity import ORD, assert_spmv_close

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def cme():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("GPU tests need a CUDA device")
    import paper_conf_ipps_maggionibl13_b200 as m
    return m


def _coo(oracle_mod, net):
    states, r, c, v = oracle_mod.enumerate_network(net)
    return len(states), r, c, v


CASES = [
    # (name, builder, order, omega, encoding knobs, compact code expected)
    ("toggle120-rcm-vi", lambda o: _coo(o, W.toggle_switch(120)), "rcm", 0.9, {}, 2),
    ("toggle90-dfs-vi", lambda o: _coo(o, W.toggle_switch(90)), "dfs", 0.9, {}, 2),
    ("schnak60-none-f64", lambda o: _coo(o, W.schnakenberg(60)), "none", 1.0, {"CME_VI": "0"}, 1),
    ("banded-w300-f64", lambda o: (40000,) + tuple(W.banded_markov(40000, 10, 300, True, seed=5)), "none", 1.0,
     {}, 1),
    ("banded-w40-rcm-f64", lambda o: (30011,) + tuple(W.banded_markov(30011, 6, 40, False, seed=6)), "rcm", 1.0,
     {}, 1),
]


@pytest.mark.parametrize("mode", ["1", "2"])   # mirrored ring / ring with a wrap per entry
@pytest.mark.parametrize("warps,stages,grid", [(30, 0, 0), (30, 2, 3), (16, 3, 5), (16, 2, 2)])
@pytest.mark.parametrize("case", CASES, ids=[c[0] for c in CASES])
def test_xw_parity(cme, oracle_mod, monkeypatch, warps, stages, grid, case, mode):
    name, make, order, omega, knobs, compact = case
    env = {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_XW": "1", "CME_XW_MODE": mode, "CME_VI2_WARPS": str(warps),
           **knobs}
    if stages:
        env["CME_VI2_STAGES"] = str(stages)
    if grid:
        env["CME_VI2_GRID"] = str(grid)
    for k, v_ in env.items():
        monkeypatch.setenv(k, v_)
    n, r, c, v = make(oracle_mod)
    A = oracle_mod.ingest(n, r, c, v)
    m = cme.Matrix(n, r, c, v).reorder(ORD[order]).pack()
    f = m.info()
    if mode == "1" and f.xwin_kb == 0:   # the mirrored ring needs the widest tile's chunks twice
        m.close()
        pytest.skip("mirrored ring does not fit this shape")
    assert f.records == 1 and f.xwin_kb > 0 and f.tma_warps == warps and f.compact == compact, \
        (f.records, f.xwin_kb, f.tma_warps, f.compact)
    if grid:
        assert f.grid <= grid   # (fewer tiles than the cap on the smallest case)
    m.set_opts(omega=omega, check_every=30, stag_tol=0.0)
    x = W.random_start(n, 21)
    assert_spmv_close(m.spmv(x), oracle_mod.jacobi_step(A, x, omega))
    p, st, it = m.solve(tol=0.0, max_iter=95)   # partial last check block
    ref = oracle_mod.jacobi_solve(A, omega=omega, tol=0.0, check_every=30, max_iter=95, stag_tol=0.0)
    assert it == ref.iters == 95 and np.abs(p - ref.p).sum() <= 1e-12
    m.close()


@pytest.mark.parametrize("mode", ["1", "2"])
@pytest.mark.parametrize("grid", [0, 4])
def test_xw_converged_and_stopped_launches(cme, oracle_mod, monkeypatch, grid, mode):
    """A converged solve: the stop decision lands inside a check block, so the
    remaining launches of the block's graph are stopped launches (their
    prologue stages hold records without x chunks and must be released)."""
    for k, v_ in {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_XW": "1", "CME_XW_MODE": mode}.items():
        monkeypatch.setenv(k, v_)
    if grid:
        monkeypatch.setenv("CME_VI2_GRID", str(grid))
    n, r, c, v = _coo(oracle_mod, W.toggle_switch(60))
    A = oracle_mod.ingest(n, r, c, v)
    m = cme.Matrix(n, r, c, v).reorder(ORD["rcm"]).pack()
    assert m.info().xwin_kb > 0
    m.set_opts(omega=0.9, check_every=100)
    p, st, it = m.solve(tol=1e-12, max_iter=100000)
    o = oracle_mod.jacobi_solve(A, omega=0.9, tol=1e-12)
    assert st == o.status == "CONVERGED" and abs(it - o.iters) <= 100
    if it != o.iters:
        o = oracle_mod.jacobi_solve(A, omega=0.9, tol=0.0, max_iter=it)
    assert np.abs(p - o.p).sum() <= 1e-10
    # a second solve on the same handle (graphs re-run, ring re-zeroed per launch)
    p2, st2, it2 = m.solve(tol=1e-12, max_iter=100000)
    assert st2 == st and it2 == it and np.array_equal(p2, p)
    m.close()


def test_xw_transient(cme, oracle_mod, monkeypatch):
    """Uniformization (NEXT-3) through the x-window kernel: its unif mode reads
    x_r from the ring too."""
    for k, v_ in {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_XW": "1", "CME_VI2_GRID": "3"}.items():
        monkeypatch.setenv(k, v_)
    n, r, c, v = _coo(oracle_mod, W.toggle_switch(50))
    A = oracle_mod.ingest(n, r, c, v)
    m = cme.Matrix(n, r, c, v).reorder(ORD["dfs"]).pack()
    assert m.info().xwin_kb > 0
    for t in (0.05, 0.5):
        pt, terms = m.transient(t)
        ref, _, _ = oracle_mod.transient(A, t)
        assert np.abs(pt - ref).sum() <= 1e-12
    m.close()


def test_xw_bit_identical_to_gather_kernel(cme, oracle_mod, monkeypatch):
    """Same records, same FMA order: the x-window kernel's SpMV equals the
    gather kernel's bit for bit (only where x comes from differs)."""
    n, r, c, v = _coo(oracle_mod, W.toggle_switch(120))
    x = W.random_start(n, 5)
    out = []
    for xw in ("0", "1"):
        for k, v_ in {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_XW": xw, "CME_VI2_WARPS": "30"}.items():
            monkeypatch.setenv(k, v_)
        m = cme.Matrix(n, r, c, v).reorder(ORD["rcm"]).pack()
        assert (m.info().xwin_kb > 0) == (xw == "1")
        m.set_opts(omega=0.9)
        out.append(m.spmv(x))
        m.close()
    assert np.array_equal(out[0], out[1])


def test_xw_auto_rule(cme, monkeypatch):
    """Auto (CME_XW unset): the x window for a random band's f64 records
    (uncoalesced gathers), not for the toggle's value-indexed records or a
    grid band's coalesced gathers."""
    for k, v_ in {"CME_TMA": "1", "CME_RESIDENT": "0"}.items():
        monkeypatch.setenv(k, v_)
    monkeypatch.delenv("CME_XW", raising=False)
    n = 400000
    r, c, v = W.banded_markov(n, 10, 1024, False, seed=2)
    m = cme.Matrix(n, r, c, v).pack()
    f = m.info()
    assert f.xwin_kb > 0 and f.records == 1 and f.compact == 1
    m.close()
    s, r, c, v = cme.cme_network_enumerate(W.schnakenberg(700))
    m = cme.Matrix(len(s), r, c, v).pack()
    assert m.info().xwin_kb == 0
    m.close()


@pytest.mark.slow
@pytest.mark.parametrize("width,mu,irr", [(1024, 10, False), (4096, 10, True)])
def test_cfg5_full_size_xw_parity(cme, oracle_mod, width, mu, irr):
    """Config 5 at the sweep's size (n = 16 M rows, 160 M entries; BASELINE
    configs[4]) on the kernel the sweep times -- the auto rule's x-window
    kernel (mirrored ring at width 1 024, the wrap mode at width 4 096): one
    SpMV on every row vs the oracle's C Jacobi step, the |a_jj|-weighted mass
    invariant, and 40 iterations of the landscape vs the oracle (all host
    threads)."""
    import os
    n = 16_000_000
    r, c, v = W.banded_markov_fast(n, mu, width, irr, seed=1)
    A = oracle_mod.ingest(n, r, c, v)
    m = cme.Matrix(n, r, c, v).pack()
    del r, c, v
    f = m.info()
    assert f.xwin_kb > 0 and f.records == 1 and f.compact == 1, (f.xwin_kb, f.records, f.compact)
    x = W.random_start(n, 23)
    m.set_opts(omega=1.0)
    y = m.spmv(x)
    assert_spmv_close(y, oracle_mod.jacobi_step(A, x, 1.0))
    d = -A.diag
    assert abs((d * y).sum() - (d * x).sum()) <= 1e-12 * (d * x).sum()
    m.set_opts(omega=1.0, check_every=20, stag_tol=0.0)
    p, st, it = m.solve(tol=0.0, max_iter=40)
    ref = oracle_mod.jacobi_solve(A, omega=1.0, tol=0.0, check_every=20, max_iter=40, stag_tol=0.0,
                                  nthreads=len(os.sched_getaffinity(0)))
    assert it == ref.iters == 40
    assert np.abs(p - ref.p).sum() <= 1e-12
    m.close()
