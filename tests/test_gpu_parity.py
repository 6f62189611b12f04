"""GPU parity: the CUDA path (through the C ABI) against the oracle.

Tolerances (north star):
* one SpMV / Jacobi application: |y_gpu - y_ora| <= 1e-13 * y_ora componentwise
  for y_ora >= 2^-1000 (absolute 1e-300 below), and L1 <= 1e-13 * ||y||_1;
* converged landscape: same (omega, tol, C, p0); stop iteration within +-C;
  ||p_gpu - p_ora||_1 <= 1e-10 (oracle re-run for exactly the GPU's count if
  the counts differ).
DESIGN.md section 6 derives why these hold (all terms non-negative: no
cancellation; expected ~5e-16 per step).
"""
import math

import numpy as np
import pytest

import workloads as W

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def cme():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("GPU tests need a CUDA device")
    import paper_conf_ipps_maggionibl13_b200 as m
    return m


def assert_spmv_close(y, ref):
    y, ref = np.asarray(y), np.asarray(ref)
    big = ref >= 2.0 ** -1000
    rel = np.abs(y[big] - ref[big]) / ref[big]
    assert rel.max(initial=0.0) <= 1e-13, rel.max()
    assert np.all(np.abs(y[~big] - ref[~big]) <= 1e-300)
    assert np.abs(y - ref).sum() <= 1e-13 * ref.sum()


NETS = [W.toggle_switch(23), W.toggle_switch(60), W.brusselator(40), W.schnakenberg(35),
        W.birth_death(100), W.schlogl(200), W.cyclic3(5), W.schnakenberg(3)]
LAYOUTS = [("none", 256, "auto", 0), ("dfs", 256, "auto", 0), ("rcm", 256, "auto", 0),
           ("rcm", 1, "never", 0), ("dfs", 1, "always", 0), ("none", 1, "auto", 1), ("rcm", 1, "auto", 2)]
ORD = {"none": 0, "dfs": 1, "rcm": 2}
BAND = {"auto": 0, "always": 1, "never": 2}


def build(cme, oracle_mod, net, order="none", window=256, band="auto", fmt=0):
    states, r, c, v = oracle_mod.enumerate_network(net)
    A = oracle_mod.ingest(len(states), r, c, v)
    m = cme.Matrix(len(states), r, c, v)
    m.reorder(ORD[order], 0)
    m.pack(fmt, window, BAND[band])
    return m, A


@pytest.mark.parametrize("net", NETS, ids=lambda n: n.name)
@pytest.mark.parametrize("layout", LAYOUTS, ids=lambda l: "-".join(map(str, l)))
@pytest.mark.parametrize("omega", [1.0, 0.9])
def test_spmv_parity(cme, oracle_mod, net, layout, omega):
    m, A = build(cme, oracle_mod, net, *layout)
    m.set_opts(omega=omega)
    x = W.random_start(A.n, 11)
    y = m.spmv(x)
    assert_spmv_close(y, oracle_mod.jacobi_step(A, x, omega))


@pytest.mark.parametrize("resident", ["-1", "1"])
def test_spmv_signed_input(cme, oracle_mod, monkeypatch, resident):
    """cme_spmv is y = M_omega x for ANY x (include/cme.h), including negative
    entries and -0.0, also on a matrix whose solves run the SMEM-resident
    kernel (which tags epochs in the sign bit and so needs x >= +0)."""
    monkeypatch.setenv("CME_RESIDENT", resident)
    m, A = build(cme, oracle_mod, W.toggle_switch(40), "rcm")
    x = W.random_start(A.n, 4) - 0.5 / A.n
    x[::7] = -0.0
    for omega in (1.0, 0.9):
        m.set_opts(omega=omega)
        y = m.spmv(x)
        ref = oracle_mod.jacobi_step(A, x, omega)
        scale = np.abs(oracle_mod.jacobi_step(A, np.abs(x), omega))   # no-cancellation magnitude
        assert np.all(np.abs(y - ref) <= 1e-13 * scale + 1e-300)
    p, st, it = m.solve(tol=1e-10, max_iter=5000)   # a solve after the signed SpMV
    assert st == "CONVERGED"
    m.close()


def test_spmv_wide_rates_and_ragged(cme, oracle_mod):
    """Config-5 generator: irregular widths, rates in [1,2), ragged last slice."""
    for n, mu, width, irr in [(1000, 10, 64, True), (777, 5, 2, False), (5000, 15, 5000, True), (33, 6, 8, True)]:
        r, c, v = W.banded_markov(n, mu, width, irr, seed=3)
        A = oracle_mod.ingest(n, r, c, v)
        for order in ("none", "rcm"):
            m = cme.Matrix(n, r, c, v).reorder(ORD[order]).pack()
            x = W.random_start(n, 5)
            assert_spmv_close(m.spmv(x), oracle_mod.jacobi_step(A, x, 1.0))


@pytest.mark.parametrize("net", NETS, ids=lambda n: n.name)
@pytest.mark.parametrize("layout", LAYOUTS[:5], ids=lambda l: "-".join(map(str, l)))
@pytest.mark.parametrize("vi", ["0", "1"])
def test_spmv_parity_compact_tma(cme, oracle_mod, monkeypatch, net, layout, vi):
    """Every SELL layout of every network through the TMA kernel on the compact
    encoding and on its value-indexed form (forced: these matrices are below
    the auto size), plus the check partials: one solve of 2 blocks against
    the oracle."""
    monkeypatch.setenv("CME_TMA", "1")
    monkeypatch.setenv("CME_RESIDENT", "0")
    monkeypatch.setenv("CME_VI", vi)
    m, A = build(cme, oracle_mod, net, *layout)
    assert m.info().kernel == 1 and m.info().compact == (1 if vi == "0" else 2)
    for omega in (1.0, 0.9):
        m.set_opts(omega=omega)
        x = W.random_start(A.n, 11)
        assert_spmv_close(m.spmv(x), oracle_mod.jacobi_step(A, x, omega))
    m.set_opts(omega=0.9, check_every=50, stag_tol=0.0, stop=cme.CME_STOP_PAPER_RESID)
    p, st, it = m.solve(tol=0.0, max_iter=100)
    ref = oracle_mod.jacobi_solve(A, omega=0.9, tol=0.0, check_every=50, max_iter=100, stag_tol=0.0)
    assert it == ref.iters and np.abs(p - ref.p).sum() <= 1e-12
    rep = m.report()
    assert rep.delta == pytest.approx(ref.delta, rel=1e-9) and rep.resid == pytest.approx(ref.resid, rel=1e-9)


@pytest.mark.parametrize("compact,vi", [("1", "1"), ("1", "0"), ("0", "0")])
def test_transient_on_tma_kernels(cme, oracle_mod, monkeypatch, compact, vi):
    """Uniformization (NEXT-3) through the TMA kernel on both encodings: the
    compact one rebuilds (A x)_r = |a_rr| ((M x)_r - x_r) from M's rows."""
    monkeypatch.setenv("CME_TMA", "1")
    monkeypatch.setenv("CME_RESIDENT", "0")
    monkeypatch.setenv("CME_COMPACT", compact)
    monkeypatch.setenv("CME_VI", vi)
    states, r, c, v = oracle_mod.enumerate_network(W.toggle_switch(50))
    A = oracle_mod.ingest(len(states), r, c, v)
    m = cme.Matrix(A.n, r, c, v).reorder(ORD["dfs"]).pack()
    assert m.info().compact == int(compact) + int(vi)
    for t in (0.05, 0.5):
        pt, terms = m.transient(t)
        ref, _, _ = oracle_mod.transient(A, t)
        assert np.abs(pt - ref).sum() <= 1e-12


def test_value_index_bit_identical_to_layout_v0(cme, oracle_mod, monkeypatch):
    """The value-indexed kernel does the layout-v0 arithmetic exactly (same
    values from the dictionary, same FMA order, row sum times inv_d): its
    SpMV and a fixed-iteration landscape are bit-identical to the v0 TMA
    kernel's."""
    monkeypatch.setenv("CME_TMA", "1")
    monkeypatch.setenv("CME_RESIDENT", "0")
    states, r, c, v = oracle_mod.enumerate_network(W.toggle_switch(90))
    x = W.random_start(len(states), 8)
    out = {}
    for enc, env in (("v0", {"CME_COMPACT": "0"}), ("vi", {"CME_COMPACT": "1", "CME_VI": "1", "CME_VI2": "0"}),
                     ("vi31", {"CME_TMA_WARPS": "31"}),   # one 1024-thread CTA per SM, 31-slice tiles
                     ("vi2", {"CME_TMA_WARPS": "16", "CME_VI2": "1", "CME_VI2_WARPS": "16"}),   # tile records
                     ("vi2w23", {"CME_VI2_WARPS": "23"}), ("vi2w30", {"CME_VI2_WARPS": "30"}),
                     ("vi2words", {"CME_VI2_WORDS": "1"})):
        for k, val in env.items():
            monkeypatch.setenv(k, val)
        m = cme.Matrix(len(states), r, c, v).reorder(cme.CME_ORDER_RCM).pack()
        m.set_opts(omega=0.9, check_every=50, stag_tol=0.0)
        p, st, it = m.solve(tol=0.0, max_iter=300)
        f = m.info()
        out[enc] = (m.spmv(x), p, f.compact, f.tma_warps, f.records)
    assert out["v0"][2] == 0 and out["vi"][2:] == (2, 16, 0) and out["vi31"][2:] == (2, 31, 0)
    assert out["vi2"][2:] == (2, 16, 1) and out["vi2w23"][2:] == (2, 23, 1) and out["vi2w30"][2:] == (2, 30, 1)
    assert out["vi2words"][2:] == (2, 30, 1)
    for enc in ("vi", "vi31", "vi2", "vi2w23", "vi2w30", "vi2words"):
        assert out["v0"][0].tobytes() == out[enc][0].tobytes(), enc
    assert out["v0"][1].tobytes() == out["vi"][1].tobytes()
    for enc in ("vi2", "vi2w23", "vi2w30", "vi2words"):   # (other grids group the check partials differently)
        assert np.abs(out["v0"][1] - out[enc][1]).sum() <= 1e-14, enc
    # 31-slice tiles group the check partials (sum y, sum |y - x|) differently,
    # so the normalising sum can differ in its last bit: same landscape to rounding
    assert np.abs(out["v0"][1] - out["vi31"][1]).sum() <= 1e-14


@pytest.mark.parametrize("vi", ["0", "1"])
def test_wide_slices_compact_and_value_index(cme, oracle_mod, monkeypatch, vi):
    """ELL widths above 8 (the chunked wide-row path of both compact kernels):
    config-5 pattern with mu = 15 and irregular degrees (rows of up to ~25
    entries), rates quantised to 8 distinct values so the value index applies."""
    monkeypatch.setenv("CME_TMA", "1")
    monkeypatch.setenv("CME_RESIDENT", "0")
    monkeypatch.setenv("CME_VI", vi)
    n = 9000
    r, c, v = W.banded_markov(n, 15, 300, True, seed=4)
    v = 1.0 + np.floor((v - 1.0) * 8.0) / 8.0          # 8 distinct rates in [1, 2)
    A = oracle_mod.ingest(n, r, c, v)
    m = cme.Matrix(n, r, c, v).pack()
    f = m.info()
    assert f.kernel == 1 and f.compact == (2 if vi == "1" else 1)
    assert m.packed()["slice_w"].max() > 8
    for omega in (1.0, 0.7):
        m.set_opts(omega=omega, check_every=20, stag_tol=0.0)
        x = W.random_start(n, 13)
        assert_spmv_close(m.spmv(x), oracle_mod.jacobi_step(A, x, omega))
    p, st, it = m.solve(tol=0.0, max_iter=60)
    ref = oracle_mod.jacobi_solve(A, omega=0.7, tol=0.0, check_every=20, max_iter=60, stag_tol=0.0)
    assert it == ref.iters and np.abs(p - ref.p).sum() <= 1e-12


def test_large_dictionary_single_dictionary_cta(cme, oracle_mod, monkeypatch):
    """A dictionary too large for two copies per SM (~14 000 distinct rates, 112 KB)
    runs the value-indexed kernel on the 31-warp single-dictionary CTA in auto
    mode (the 100M-state toggle's case: 14.1K distinct rates), with oracle parity."""
    monkeypatch.setenv("CME_TMA", "1")
    monkeypatch.setenv("CME_RESIDENT", "0")
    n = 60000
    r, c, v = W.banded_markov(n, 6, 200, True, seed=9)
    v = 1.0 + np.floor((v - 1.0) * 14000.0) / 14000.0    # ~14 000 distinct rates in [1, 2)
    A = oracle_mod.ingest(n, r, c, v)
    m = cme.Matrix(n, r, c, v).pack()
    f = m.info()
    # single-dictionary CTA: the tile-record kernel's 30 consumer warps (or
    # sell_vi_kernel's 31 when the records are off)
    assert f.kernel == 1 and f.compact == 2 and (f.tma_warps, f.records) in ((30, 1), (31, 0))
    for omega in (1.0, 0.8):
        m.set_opts(omega=omega, check_every=20, stag_tol=0.0)
        x = W.random_start(n, 17)
        assert_spmv_close(m.spmv(x), oracle_mod.jacobi_step(A, x, omega))
    p, st, it = m.solve(tol=0.0, max_iter=60)
    ref = oracle_mod.jacobi_solve(A, omega=0.8, tol=0.0, check_every=20, max_iter=60, stag_tol=0.0)
    assert it == ref.iters and np.abs(p - ref.p).sum() <= 1e-12


def test_compact_fallback_wide_offsets(cme, oracle_mod, monkeypatch):
    """A transition spanning > 32767 states has no int16 offset: the TMA kernel
    keeps layout v0 (compact = 0) and stays exact."""
    monkeypatch.setenv("CME_TMA", "1")
    monkeypatch.setenv("CME_RESIDENT", "0")
    n = 70000
    r, c, v = W.banded_markov(n, 6, 40000, True, seed=9)
    A = oracle_mod.ingest(n, r, c, v)
    m = cme.Matrix(n, r, c, v).pack()
    assert m.info().kernel == 1 and m.info().compact == 0
    # rates in [1, 2) are all distinct: the compact-encodable band has no value index either
    r2, c2, v2 = W.banded_markov(n, 6, 300, True, seed=9)
    A2 = oracle_mod.ingest(n, r2, c2, v2)
    m2 = cme.Matrix(n, r2, c2, v2).pack()
    assert m2.info().kernel == 1 and m2.info().compact == 1
    x2 = W.random_start(n, 6)
    assert_spmv_close(m2.spmv(x2), oracle_mod.jacobi_step(A2, x2, 1.0))
    x = W.random_start(n, 5)
    assert_spmv_close(m.spmv(x), oracle_mod.jacobi_step(A, x, 1.0))


def solve_both(cme, oracle_mod, m, A, omega, tol, C=100, max_iter=200000, p0=None, stag=1e-10):
    m.set_opts(omega=omega, check_every=C, stag_tol=stag)
    p, st, it = m.solve(p0=p0, tol=tol, max_iter=max_iter)
    r = oracle_mod.jacobi_solve(A, p0=p0, omega=omega, tol=tol, check_every=C, max_iter=max_iter,
                                stag_tol=stag)
    return p, st, it, r


@pytest.mark.parametrize("net,omega", [(W.birth_death(100), 0.9), (W.toggle_switch(40), 0.9),
                                       (W.schnakenberg(30, 8, 1, 5, 1, 0.01), 1.0),
                                       (W.cyclic3(6), 0.5), (W.schlogl(120, c3=20.0, c4=1.0), 0.9)],
                         ids=lambda x: getattr(x, "name", str(x)))
@pytest.mark.parametrize("layout", [("none", 256, "auto", 0), ("rcm", 1, "never", 0), ("dfs", 256, "auto", 2)],
                         ids=lambda l: "-".join(map(str, l)))
def test_landscape_parity(cme, oracle_mod, net, omega, layout):
    m, A = build(cme, oracle_mod, net, *layout)
    p, st, it, r = solve_both(cme, oracle_mod, m, A, omega, 1e-12)
    assert st == r.status == "CONVERGED"
    assert abs(it - r.iters) <= 100
    if it != r.iters:
        r = oracle_mod.jacobi_solve(A, omega=omega, tol=0.0, max_iter=it)
    assert np.abs(p - r.p).sum() <= 1e-10
    assert abs(p.sum() - 1.0) < 1e-13 and p.min() >= 0


def test_closed_forms(cme, oracle_mod):
    m, A = build(cme, oracle_mod, W.birth_death(100))
    m.set_opts(omega=0.9)
    p, st, it = m.solve(tol=1e-14, max_iter=400000)
    logs = np.array([x * math.log(10.0) - math.lgamma(x + 1) for x in range(101)])
    pi = np.exp(logs - logs.max()); pi /= pi.sum()
    assert st == "CONVERGED" and np.abs(p - pi).sum() < 1e-11
    net = W.schnakenberg(40, 8.0, 1.0, 5.0, 1.0, 0.01)
    m = cme.Matrix.from_network(net).reorder(cme.CME_ORDER_RCM).pack()
    p, st, it = m.solve(tol=1e-15, max_iter=400000)
    logs = np.array([x * math.log(8.0) - math.lgamma(x + 1) + y * math.log(5.0) - math.lgamma(y + 1)
                     for x, y in m.states])
    pi = np.exp(logs - logs.max()); pi /= pi.sum()
    assert st == "CONVERGED" and np.abs(p - pi).sum() < 1e-12


def test_stagnation_on_periodic_chain(cme, oracle_mod):
    m, A = build(cme, oracle_mod, W.birth_death(100))
    assert m.info().period == 2 and m.info().omega == 0.9
    p, st, it, r = solve_both(cme, oracle_mod, m, A, 1.0, 1e-14)
    assert st == r.status == "STAGNATED" and it == r.iters
    m, A = build(cme, oracle_mod, W.cyclic3(3))
    assert m.info().period == 3
    p, st, it, r = solve_both(cme, oracle_mod, m, A, 1.0, 1e-14)
    assert st == r.status == "STAGNATED"


def test_paper_residual_stop(cme, oracle_mod):
    m, A = build(cme, oracle_mod, W.toggle_switch(30), "rcm")
    m.set_opts(omega=0.9, stop=cme.CME_STOP_PAPER_RESID)
    p, st, it = m.solve(tol=1e-8, max_iter=100000)
    r = oracle_mod.jacobi_solve(A, omega=0.9, tol=1e-8, max_iter=100000, stop_mode=1)
    assert st == r.status == "CONVERGED" and abs(it - r.iters) <= 100
    rep = m.report()
    assert rep.resid <= 1e-8
    if it == r.iters:
        assert rep.resid == pytest.approx(r.resid, rel=1e-6)


@pytest.mark.parametrize("C", [1, 7, 100])
def test_max_iter_partial_blocks_and_p0(cme, oracle_mod, C):
    m, A = build(cme, oracle_mod, W.toggle_switch(25), "rcm", 256)
    p0 = W.random_start(A.n, 2) * 3.0
    for max_iter in (0, 1, 5, 250):
        p, st, it, r = solve_both(cme, oracle_mod, m, A, 0.9, 0.0, C=C, max_iter=max_iter, p0=p0, stag=0.0)
        assert st == r.status == "NOT_CONVERGED" and it == r.iters == max_iter
        assert np.abs(p - r.p).sum() <= 1e-12


def test_device_pointers_and_streams(cme, oracle_mod):
    import torch
    m, A = build(cme, oracle_mod, W.schnakenberg(50), "rcm")
    s = torch.cuda.Stream()
    m.set_opts(omega=1.0, stream=s.cuda_stream)
    p0 = torch.tensor(W.random_start(A.n, 9), device="cuda")
    out = torch.empty(A.n, dtype=torch.float64, device="cuda")
    p, st, it = m.solve(p0=p0, tol=1e-12, max_iter=100000, p_out=out)
    r = oracle_mod.jacobi_solve(A, p0=p0.cpu().numpy(), omega=1.0, tol=1e-12)
    assert st == r.status and abs(it - r.iters) <= 100
    if it != r.iters:
        r = oracle_mod.jacobi_solve(A, p0=p0.cpu().numpy(), omega=1.0, tol=0.0, max_iter=it)
    assert np.abs(out.cpu().numpy() - r.p).sum() <= 1e-10
    x = torch.tensor(W.random_start(A.n, 4), device="cuda")
    y = torch.empty_like(x)
    cme.cme_spmv(m.h, A.n, x, y)
    assert_spmv_close(y.cpu().numpy(), oracle_mod.jacobi_step(A, x.cpu().numpy(), 1.0))


def test_resident_run_api(cme, oracle_mod):
    m, A = build(cme, oracle_mod, W.toggle_switch(40), "rcm")
    m.set_opts(omega=0.9, check_every=50)
    cme.cme_solver_load(m.h, A.n, None)
    cme.cme_solver_run(m.h, 3)
    p = np.empty(A.n)
    cme.cme_solver_fetch(m.h, A.n, p)
    r = oracle_mod.jacobi_solve(A, omega=0.9, tol=0.0, check_every=50, max_iter=150, stag_tol=0.0)
    assert np.abs(p - r.p).sum() <= 1e-12 and m.report().iters == 150


def test_invalid_p0(cme, oracle_mod):
    m, A = build(cme, oracle_mod, W.toggle_switch(10))
    bad = np.ones(A.n); bad[3] = -1.0
    with pytest.raises(cme.CmeError) as e:
        m.solve(p0=bad)
    assert e.value.status == cme.CME_ERR_INVALID_ARG


@pytest.mark.slow
def test_cfg2_toggle_landscape(cme, oracle_mod):
    """Config 2: toggle N=224, omega 0.9, tol 1e-12, bimodal landscape."""
    net = W.toggle_switch(224)
    m = cme.Matrix.from_network(net).reorder(cme.CME_ORDER_RCM).pack()
    A = oracle_mod.network_csr(net)
    m.set_opts(omega=0.9)
    p, st, it = m.solve(tol=1e-12, max_iter=100000)
    r = oracle_mod.jacobi_solve(A, omega=0.9, tol=1e-12, nthreads=8)
    assert st == r.status == "CONVERGED" and abs(it - r.iters) <= 100
    if it != r.iters:
        r = oracle_mod.jacobi_solve(A, omega=0.9, tol=0.0, max_iter=it, nthreads=8)
    assert np.abs(p - r.p).sum() <= 1e-10
    S = m.states
    onoff = p[(S[:, 0] >= 20) & (S[:, 1] < 5)].sum()
    assert 0.40 < onoff < 0.50


@pytest.mark.slow
def test_cfg3a_schnakenberg_closed_form_at_scale(cme):
    """Config 3a: n = 2,003,001 (Table I size), detailed balance -> product Poisson."""
    net = W.schnakenberg(2000)
    m = cme.Matrix.from_network(net).pack()
    assert m.info().n == 2003001 and m.info().nnz == 14001003
    p, st, it = m.solve(tol=1e-14, max_iter=2_000_000)
    assert st == "CONVERGED"
    S = m.states.astype(np.float64)
    a, b = 500.0, 400.0
    from scipy.special import gammaln
    logs = S[:, 0] * math.log(a) - gammaln(S[:, 0] + 1) + S[:, 1] * math.log(b) - gammaln(S[:, 1] + 1)
    pi = np.exp(logs - logs.max())
    pi /= pi.sum()
    assert np.abs(p - pi).sum() <= 1e-10


def test_nccl_one_rank_distributed_path(cme, oracle_mod):
    """The distributed code path (NCCL allgather of the check record, segment
    broadcast of the output) with a 1-rank communicator on this GPU must give
    the single-GPU result.  >= 2 ranks need >= 2 GPUs (tests/test_partition_gloo.py
    covers the multi-rank protocol on CPU)."""
    import torch
    import paper_conf_ipps_maggionibl13_b200 as m
    net = W.toggle_switch(45)
    states, r, c, v = oracle_mod.enumerate_network(net)
    A = oracle_mod.ingest(len(states), r, c, v)
    ref = m.Matrix(A.n, r, c, v).reorder(m.CME_ORDER_RCM).pack()
    ref.set_opts(omega=0.9)
    p_ref, st_ref, it_ref = ref.solve(tol=1e-12)
    uid = m.cme_comm_unique_id()
    comm = m.cme_comm_init(1, 0, uid, torch.cuda.current_device())
    d = m.Matrix(A.n, r, c, v).reorder(m.CME_ORDER_RCM)
    d.pack(device=m.CME_DEVICE_HOST_ONLY)
    m.cme_matrix_distribute(d.h, comm)
    d.set_opts(omega=0.9)
    p, st, it = d.solve(tol=1e-12)
    assert st == st_ref == "CONVERGED" and it == it_ref
    assert np.abs(p - p_ref).sum() <= 1e-14
    x = W.random_start(A.n, 3)
    assert_spmv_close(d.spmv(x), oracle_mod.jacobi_step(A, x, 0.9))
    d.close()
    m.cme_comm_destroy(comm)


@pytest.mark.parametrize("knobs", [{"CME_TMA": "0", "CME_RESIDENT": "0"}, {"CME_TMA": "1", "CME_RESIDENT": "0"},
                                   {"CME_TMA": "1", "CME_TMA_WARPS": "8", "CME_RESIDENT": "0"},
                                   {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_COMPACT": "0"},
                                   {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_VI": "0"},
                                   {"CME_TMA": "1", "CME_TMA_WARPS": "31", "CME_VI": "1", "CME_RESIDENT": "0"},
                                   {"CME_RESIDENT": "1"}],
                         ids=lambda k: ",".join(f"{a}={b}" for a, b in k.items()))
@pytest.mark.parametrize("net,order,omega", [(W.toggle_switch(70), "rcm", 0.9), (W.schnakenberg(120), "none", 1.0),
                                             (W.brusselator(90), "dfs", 0.7)], ids=lambda x: getattr(x, "name", str(x)))
def test_every_step_kernel(cme, oracle_mod, monkeypatch, knobs, net, order, omega):
    """Each step kernel (register SELL, TMA-staged SELL with 16/8 consumer
    warps, SMEM-resident persistent with epoch-tagged iterates) forced on the
    same problems: per-step parity and a fixed-iteration landscape (C = 7
    exercises odd block parity and, with max_iter = 250, a partial final block)."""
    for k, v in knobs.items():
        monkeypatch.setenv(k, v)
    states, r, c, v = oracle_mod.enumerate_network(net)
    A = oracle_mod.ingest(len(states), r, c, v)
    m = cme.Matrix(A.n, r, c, v).reorder(ORD[order]).pack()
    f = m.info()
    expect = 3 if knobs.get("CME_RESIDENT") == "1" else 1 if knobs["CME_TMA"] == "1" else 0
    assert f.kernel == expect
    # the TMA kernel streams the value-indexed compact encoding (2) unless
    # CME_VI=0 (compact, 1) or CME_COMPACT=0 (layout v0, 0)
    want = 0 if expect != 1 or knobs.get("CME_COMPACT") == "0" else 1 if knobs.get("CME_VI") == "0" else 2
    assert f.compact == want
    m.set_opts(omega=omega, check_every=7, stag_tol=0.0)
    x = W.random_start(A.n, 21)
    assert_spmv_close(m.spmv(x), oracle_mod.jacobi_step(A, x, omega))
    p, st, it = m.solve(tol=0.0, max_iter=250)
    ref = oracle_mod.jacobi_solve(A, omega=omega, tol=0.0, check_every=7, max_iter=250, stag_tol=0.0)
    assert it == ref.iters == 250 and np.abs(p - ref.p).sum() <= 1e-12
    p, st, it = m.solve(tol=1e-11, max_iter=100000)
    ref = oracle_mod.jacobi_solve(A, omega=omega, tol=1e-11, check_every=7, max_iter=100000, stag_tol=0.0)
    assert st == ref.status and abs(it - ref.iters) <= 7


@pytest.fixture(scope="module")
def cfg4(cme, oracle_mod):
    """The bench workload (configs[3]: toggle N=3164, n = 20,015,468), packed
    exactly as bench.py packs it, and the oracle's own enumeration + CSR."""
    net = W.config_network("cfg4_toggle_20m")
    m = cme.Matrix.from_network(net).reorder(cme.CME_ORDER_RCM).pack()
    A = oracle_mod.network_csr(net)
    yield m, A
    m.close()


@pytest.mark.slow
def test_cfg4_full_size_parity(cme, oracle_mod, cfg4):
    """The bench workload itself (configs[3]: toggle N=3164, n = 20,015,468, RCM,
    the kernel bench.py times): one SpMV on every row, the |d|-weighted mass
    invariant, and 300 iterations of the landscape against the
    oracle's own enumeration + CSR Jacobi (16 host threads)."""
    import os
    m, A = cfg4
    info = m.info()
    assert info.n == 20015468 and info.nnz == 120042194 and info.kernel == 1 and info.compact == 2
    x = W.random_start(A.n, 17)
    m.set_opts(omega=1.0)
    y = m.spmv(x)
    assert_spmv_close(y, oracle_mod.jacobi_step(A, x, 1.0))
    d = -A.diag
    assert abs((d * y).sum() - (d * x).sum()) <= 1e-12 * (d * x).sum()
    m.set_opts(omega=0.9, stag_tol=0.0)
    p, st, it = m.solve(tol=0.0, max_iter=300)
    ref = oracle_mod.jacobi_solve(A, omega=0.9, tol=0.0, max_iter=300, stag_tol=0.0,
                                  nthreads=len(os.sched_getaffinity(0)))
    assert it == ref.iters == 300
    assert np.abs(p - ref.p).sum() <= 1e-10


@pytest.mark.slow
def test_cfg4_converged_landscape(cme, oracle_mod, cfg4):
    """North-star landscape parity at the headline scale (SURVEY 8(c5)(iii),
    P:L111-125): cfg4 solved to tol 1e-12 from uniform p0 with C = 100 by the
    kernel bench.py times (value-indexed TMA kernel, info.compact == 2) and by
    the oracle (plain C CSR Jacobi, all host cores).  Same stop iteration
    within +-C; if the counts differ the oracle is re-run for exactly the GPU's
    count; then ||p_gpu - p_oracle||_1 <= 1e-10."""
    import os
    m, A = cfg4
    info = m.info()
    assert info.kernel == 1 and info.compact == 2
    m.set_opts(omega=0.9, check_every=100, stag_tol=1e-10, stop=cme.CME_STOP_DELTA_L1)
    p, st, it = m.solve(tol=1e-12, max_iter=200000)
    nt = len(os.sched_getaffinity(0))
    ref = oracle_mod.jacobi_solve(A, omega=0.9, tol=1e-12, check_every=100, max_iter=200000, nthreads=nt)
    assert st == ref.status == "CONVERGED", (st, ref.status)
    assert abs(it - ref.iters) <= 100, (it, ref.iters)
    if it != ref.iters:
        ref = oracle_mod.jacobi_solve(A, omega=0.9, tol=0.0, check_every=100, max_iter=it, stag_tol=0.0,
                                      nthreads=nt)
    err = float(np.abs(p - ref.p).sum())
    assert err <= 1e-10, err
    assert abs(p.sum() - 1.0) <= 1e-12 and np.all(p >= 0)


def directed_ring(n, hops=(1, 5), rates=(1.0, 0.5)):
    """Off-diagonal COO of a one-way ring: j -> j+h (mod n) for each hop h.
    Column j's entries are read by rows ahead of it only, so with contiguous
    row blocks every block is read by the NEXT block but reads only the
    PREVIOUS one: the resident kernel's WAR protection needs its probes."""
    j = np.arange(n, dtype=np.int64)
    rows = np.concatenate([(j + h) % n for h in hops]).astype(np.int32)
    cols = np.concatenate([j for _ in hops]).astype(np.int32)
    vals = np.concatenate([np.full(n, r) for r in rates])
    order = np.lexsort((rows, cols))
    return rows[order], cols[order], vals[order]


@pytest.mark.parametrize("width", [16, 5000, "ring"])
def test_resident_dependency_ranges(cme, oracle_mod, monkeypatch, width):
    """SMEM-resident kernel on config-5 generator matrices whose column reach
    is narrow (a few neighbour CTAs) or global (every CTA depends on every
    other): SpMV, a fixed-iteration landscape with a partial last block, and
    a solve to convergence, all against the oracle; the free-running API
    (cme_solver_load/run/fetch) continues across launches."""
    monkeypatch.setenv("CME_RESIDENT", "1")
    n = 20000
    r, c, v = directed_ring(n) if width == "ring" else W.banded_markov(n, 10, width, True, seed=5)
    A = oracle_mod.ingest(n, r, c, v)
    m = cme.Matrix(n, r, c, v).pack()
    f = m.info()
    assert f.kernel == 3 and f.grid > 1
    x = W.random_start(n, 2)
    m.set_opts(omega=0.8, check_every=10, stag_tol=0.0)
    assert_spmv_close(m.spmv(x), oracle_mod.jacobi_step(A, x, 0.8))
    p, st, it = m.solve(p0=x, tol=0.0, max_iter=95)
    ref = oracle_mod.jacobi_solve(A, p0=x, omega=0.8, tol=0.0, check_every=10, max_iter=95, stag_tol=0.0)
    assert st == ref.status == "NOT_CONVERGED" and it == ref.iters == 95
    assert np.abs(p - ref.p).sum() <= 1e-12
    # width 16 mixes too slowly to converge in 20000 iterations (both sides
    # report NOT_CONVERGED); width 5000 converges in a few hundred
    p, st, it = m.solve(p0=x, tol=1e-12, max_iter=20000)
    ref = oracle_mod.jacobi_solve(A, p0=x, omega=0.8, tol=1e-12, check_every=10, max_iter=20000, stag_tol=0.0)
    assert st == ref.status and abs(it - ref.iters) <= 10
    assert st == ("NOT_CONVERGED" if width == 16 else st)
    if it != ref.iters:
        ref = oracle_mod.jacobi_solve(A, p0=x, omega=0.8, tol=0.0, check_every=10, max_iter=it, stag_tol=0.0)
    assert np.abs(p - ref.p).sum() <= 1e-10
    # free-running: 3 blocks, then 4 more in a second launch == 70 iterations
    cme.cme_solver_load(m.h, n, x)
    cme.cme_solver_run(m.h, 3)
    cme.cme_solver_run(m.h, 4)
    q = np.empty(n)
    cme.cme_solver_fetch(m.h, n, q)
    ref = oracle_mod.jacobi_solve(A, p0=x, omega=0.8, tol=0.0, check_every=10, max_iter=70, stag_tol=0.0)
    assert np.abs(q - ref.p).sum() <= 1e-12


ABLATION_ARMS = [("sell256", dict(fmt=3, window=1)), ("random-order", dict(perm=True)),
                 ("global-window", dict(window=1 << 30)), ("ell", dict(fmt=1, window=1)),
                 ("csr", dict(fmt=2, window=1))]


@pytest.mark.parametrize("arm,kw", ABLATION_ARMS, ids=[a for a, _ in ABLATION_ARMS])
@pytest.mark.parametrize("net", [W.toggle_switch(60), W.schnakenberg(35), W.brusselator(40)], ids=lambda n: n.name)
@pytest.mark.parametrize("tma", ["0", "1"])
def test_ablation_arms_on_gpu(cme, oracle_mod, monkeypatch, arm, kw, net, tma):
    """NEXT-2 format/ordering arms of Tables II-III and sec. VII-C
    through the GPU path, against the oracle: 256-row block-sliced ELL ([5],
    P:L159), a seeded random ordering (the locality stress of P:L225), the
    global rearrangement window (pJDS-like, window >= n), plain ELL and CSR.
    SpMV per step, a fixed-iteration landscape and a solve to convergence."""
    assert cme.CME_FMT_SELL256 == 3 and cme.CME_FMT_ELL == 1 and cme.CME_FMT_CSR == 2
    monkeypatch.setenv("CME_TMA", tma)
    monkeypatch.setenv("CME_RESIDENT", "0")
    states, r, c, v = oracle_mod.enumerate_network(net)
    A = oracle_mod.ingest(len(states), r, c, v)
    m = cme.Matrix(A.n, r, c, v)
    if kw.get("perm"):
        m.set_permutation(np.random.default_rng(9).permutation(A.n).astype(np.int32))
    m.pack(kw.get("fmt", 0), kw.get("window", 256), 0)
    omega = 0.9 if oracle_mod.period(A) != 1 else 1.0
    m.set_opts(omega=omega, check_every=40, stag_tol=0.0)
    x = W.random_start(A.n, 6)
    assert_spmv_close(m.spmv(x), oracle_mod.jacobi_step(A, x, omega))
    p, st, it = m.solve(tol=0.0, max_iter=200)
    ref = oracle_mod.jacobi_solve(A, omega=omega, tol=0.0, check_every=40, max_iter=200, stag_tol=0.0)
    assert it == ref.iters == 200 and np.abs(p - ref.p).sum() <= 1e-12
    p, st, it = m.solve(tol=1e-11, max_iter=30000)   # toggle converges; the others stop at max_iter
    ref = oracle_mod.jacobi_solve(A, omega=omega, tol=1e-11, check_every=40, max_iter=30000, stag_tol=0.0)
    assert st == ref.status and abs(it - ref.iters) <= 40
    if it != ref.iters:
        ref = oracle_mod.jacobi_solve(A, omega=omega, tol=0.0, check_every=40, max_iter=it, stag_tol=0.0)
    assert np.abs(p - ref.p).sum() <= 1e-10
    m.close()


@pytest.mark.parametrize("words", ["0", "1"])
@pytest.mark.parametrize("warps,stages,grid", [(16, 2, 3), (23, 2, 5), (30, 3, 2), (23, 4, 7)])
@pytest.mark.parametrize("net,order,omega", [(W.toggle_switch(120), "rcm", 0.9), (W.toggle_switch(90), "dfs", 0.9)],
                         ids=lambda x: getattr(x, "name", str(x)))
def test_vi2_ring_wraps(cme, oracle_mod, monkeypatch, warps, stages, grid, net, order, omega, words):
    """Tile-record kernel (sell_vi2_kernel) with its grid capped to a few CTAs,
    so every CTA streams dozens of tiles through its 2-4 stage ring (the ring
    reuse and mbarrier parity logic that a full grid never exercises on a
    small matrix): SpMV and a fixed-iteration landscape vs the oracle."""
    for k, v_ in {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_VI2_WARPS": str(warps), "CME_VI2_STAGES": str(stages),
                  "CME_VI2_GRID": str(grid), "CME_VI2_WORDS": words}.items():
        monkeypatch.setenv(k, v_)
    states, r, c, v = oracle_mod.enumerate_network(net)
    A = oracle_mod.ingest(len(states), r, c, v)
    m = cme.Matrix(A.n, r, c, v).reorder(ORD[order]).pack()
    f = m.info()
    assert f.records == 1 and f.tma_warps == warps and f.grid == grid
    m.set_opts(omega=omega, check_every=30, stag_tol=0.0)
    x = W.random_start(A.n, 12)
    assert_spmv_close(m.spmv(x), oracle_mod.jacobi_step(A, x, omega))
    p, st, it = m.solve(tol=0.0, max_iter=90)
    ref = oracle_mod.jacobi_solve(A, omega=omega, tol=0.0, check_every=30, max_iter=90, stag_tol=0.0)
    assert it == ref.iters == 90 and np.abs(p - ref.p).sum() <= 1e-12
    m.close()


@pytest.mark.parametrize("steps", [2, 3])
@pytest.mark.parametrize("warps,grid,lag", [(30, 0, -1), (16, 3, 0)])
@pytest.mark.parametrize("net,order,omega", [(W.toggle_switch(120), "rcm", 0.9), (W.toggle_switch(90), "dfs", 0.9)],
                         ids=lambda x: getattr(x, "name", str(x)))
def test_wavefront_passes(cme, oracle_mod, monkeypatch, steps, warps, grid, lag, net, order, omega):
    """Wavefront s-step kernel (sell_wf_kernel): check
    blocks run as passes of s Jacobi steps whose later steps wait on per-tile
    completion counters.  Capped grids (3 or 5 CTAs) and a minimal lag make
    the dependency waits and the ring reuse happen on every item; C = 40 with
    s = 3 leaves a 1-step remainder per block on the single-step kernel, and
    max_iter = 95 a partial last block.  Fixed-iteration landscapes and a
    converged solve vs the oracle."""
    env = {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_VI2_WARPS": str(warps), "CME_WF": str(steps)}
    if grid:
        env["CME_VI2_GRID"] = str(grid)
    if lag >= 0:
        env["CME_WF_LAG"] = str(lag)
    for k, v_ in env.items():
        monkeypatch.setenv(k, v_)
    states, r, c, v = oracle_mod.enumerate_network(net)
    A = oracle_mod.ingest(len(states), r, c, v)
    m = cme.Matrix(A.n, r, c, v).reorder(ORD[order]).pack()
    f = m.info()
    assert f.records == 1 and f.wf_steps == steps and f.tma_warps == warps and f.wf_lag > 0
    if grid:
        assert f.grid == grid
    m.set_opts(omega=omega, check_every=30, stag_tol=0.0)
    for max_iter in (90, 95):
        p, st, it = m.solve(tol=0.0, max_iter=max_iter)
        ref = oracle_mod.jacobi_solve(A, omega=omega, tol=0.0, check_every=30, max_iter=max_iter, stag_tol=0.0)
        assert it == ref.iters == max_iter and np.abs(p - ref.p).sum() <= 1e-12, (max_iter, np.abs(p - ref.p).sum())
    m.set_opts(omega=omega, check_every=40, stag_tol=0.0)
    p, st, it = m.solve(tol=1e-9, max_iter=20000)
    ref = oracle_mod.jacobi_solve(A, omega=omega, tol=1e-9, check_every=40, max_iter=20000, stag_tol=0.0)
    assert st == ref.status and abs(it - ref.iters) <= 40
    if it != ref.iters:
        ref = oracle_mod.jacobi_solve(A, omega=omega, tol=0.0, check_every=40, max_iter=it, stag_tol=0.0)
    assert np.abs(p - ref.p).sum() <= 1e-10
    m.close()


def test_wavefront_bit_identical_steps(cme, monkeypatch):
    """Between checks the wavefront passes apply the same per-row arithmetic
    as the single-step kernel: with no check inside the run (C larger than
    max_iter) and the same final normalisation, 24 iterations as 12 passes of
    2 / 8 passes of 3 / 6 of 4 give the single-step result to the last bit up
    to the final 1/sum scale (whose summation order differs)."""
    net = W.toggle_switch(150)
    states, r, c, v = cme.cme_network_enumerate(net)
    outs = {}
    for s in ("0", "2", "3", "4"):
        for k, v_ in {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_WF": s}.items():
            monkeypatch.setenv(k, v_)
        m = cme.Matrix(len(states), r, c, v).reorder(2).pack()
        assert m.info().wf_steps == (int(s) if s != "0" else 0)
        m.set_opts(omega=0.9, check_every=24, stag_tol=0.0)
        p, st, it = m.solve(tol=0.0, max_iter=24, p0=W.random_start(len(states), 5))
        assert it == 24
        outs[s] = p
        m.close()
    for s in ("2", "3", "4"):
        ratio = outs[s] / outs["0"]      # one common scale: x_24 itself is identical
        assert np.abs(ratio / ratio[0] - 1.0).max() <= 1e-15, (s, np.abs(ratio / ratio[0] - 1.0).max())
        assert abs(ratio[0] - 1.0) <= 1e-13


@pytest.mark.parametrize("warps,grid", [(30, 0), (16, 3), (30, 2)])
@pytest.mark.parametrize("net,order,omega", [(W.schnakenberg(60), "none", 1.0), (W.brusselator(70), "dfs", 0.9),
                                             (W.schlogl(300), "rcm", 0.9)],
                         ids=lambda x: getattr(x, "name", str(x)))
def test_f64_records_bit_identical_to_compact(cme, oracle_mod, monkeypatch, warps, grid, net, order, omega):
    """Tile records of the f64 compact encoding (sell_vi2_kernel ENC = 2:
    networks without a value index, e.g. Schnakenberg / Brusselator with ~10^6
    distinct rates at scale) run sell_cpt_kernel's arithmetic: SpMV and a
    fixed-iteration landscape bit-identical to CME_REC = 0 (the compact
    kernel) with the same check grid, and vs the oracle; capped grids wrap the
    ring many times."""
    states, r, c, v = oracle_mod.enumerate_network(net)
    A = oracle_mod.ingest(len(states), r, c, v)
    x = W.random_start(A.n, 21)
    outs = {}
    for rec in ("0", "1"):
        env = {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_VI": "0", "CME_REC": rec,   # (records are opt-in)
               "CME_XW": "0"}   # (the x-window kernel has its own tests: test_xw.py)
        if rec == "1":
            env["CME_VI2_WARPS"] = str(warps)
            if grid:
                env["CME_VI2_GRID"] = str(grid)
        for k, v_ in env.items():
            monkeypatch.setenv(k, v_)
        for k in ("CME_VI2_WARPS", "CME_VI2_GRID"):
            if k not in env:
                monkeypatch.delenv(k, raising=False)
        m = cme.Matrix(A.n, r, c, v).reorder(ORD[order]).pack()
        f = m.info()
        assert f.compact == 1 and f.records == int(rec), (f.compact, f.records)
        if rec == "1":
            assert f.tma_warps == warps and (not grid or f.grid <= grid)
        m.set_opts(omega=omega, check_every=25, stag_tol=0.0)
        y = m.spmv(x)
        assert_spmv_close(y, oracle_mod.jacobi_step(A, x, omega))
        p, st, it = m.solve(tol=0.0, max_iter=75)
        ref = oracle_mod.jacobi_solve(A, omega=omega, tol=0.0, check_every=25, max_iter=75, stag_tol=0.0)
        assert it == ref.iters == 75 and np.abs(p - ref.p).sum() <= 1e-12
        outs[rec] = (y, p)
        m.close()
    assert np.array_equal(outs["0"][0], outs["1"][0])   # same per-row arithmetic
