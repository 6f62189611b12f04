"""Pins for the oracle's transient solver (uniformization; P:L277 future work).

* birth-death from x = 0: the M/M/inf queue is Poisson(lam (1 - e^{-mu t}) / mu)
  at every t (truncation at N = 100 is immaterial for a mean <= 10);
* scipy.linalg.expm(A t) @ p0 (Pade, a different algorithm) on small networks;
* t = 0 returns p0; large t returns the LU steady state; mass is conserved.
"""
import math

import numpy as np
import pytest
from scipy.linalg import expm

import workloads as W


@pytest.mark.parametrize("t", [0.05, 0.5, 2.0, 8.0])
def test_birth_death_poisson_closed_form(oracle_mod, t):
    A = oracle_mod.network_csr(W.birth_death(100, 10.0, 1.0))
    p, terms, lam = oracle_mod.transient(A, t)
    m = 10.0 * (1.0 - math.exp(-t))
    ref = np.array([math.exp(-m + x * math.log(m) - math.lgamma(x + 1)) for x in range(101)])
    assert lam == 109.0 and terms > lam * t     # max outflow: lam + mu*99 at x = 99
    assert np.abs(p - ref).sum() < 1e-12


@pytest.mark.parametrize("net,t", [(W.toggle_switch(8), 0.3), (W.cyclic3(4), 1.7),
                                   (W.schnakenberg(10, 8, 1, 5, 1, 0.01), 0.9)], ids=lambda x: getattr(x, "name", str(x)))
def test_matches_expm(oracle_mod, net, t):
    A = oracle_mod.network_csr(net)
    p0 = W.random_start(A.n, 7); p0 /= p0.sum()
    p, terms, lam = oracle_mod.transient(A, t, p0=p0)
    ref = expm(A.dense() * t) @ p0
    assert np.abs(p - ref).sum() < 1e-12
    assert abs(p.sum() - 1.0) < 1e-13


def test_limits(oracle_mod):
    A = oracle_mod.network_csr(W.toggle_switch(6))
    p0 = W.random_start(A.n, 2); p0 /= p0.sum()
    p, terms, _ = oracle_mod.transient(A, 0.0, p0=p0)
    assert terms == 1 and np.array_equal(p, p0)
    p, terms, _ = oracle_mod.transient(A, 2000.0, p0=p0)
    assert np.abs(p - oracle_mod.lu_steady(A)).sum() < 1e-10
    e0 = np.zeros(A.n); e0[0] = 1.0
    pa, _, _ = oracle_mod.transient(A, 0.4)          # default start: all mass on state 0 (x0)
    pb, _, _ = oracle_mod.transient(A, 0.4, p0=e0)
    assert np.array_equal(pa, pb)


# ------------------------------------------------------------------ GPU -------
@pytest.mark.gpu
@pytest.mark.parametrize("net,order,t", [(W.birth_death(100, 10.0, 1.0), "none", 0.7),
                                         (W.toggle_switch(40), "rcm", 0.25), (W.schnakenberg(60), "none", 0.05),
                                         (W.cyclic3(9), "dfs", 3.0)], ids=lambda x: getattr(x, "name", str(x)))
@pytest.mark.parametrize("knobs", [{"CME_TMA": "0"}, {"CME_TMA": "1"}], ids=lambda k: str(k))
def test_gpu_transient_parity(oracle_mod, monkeypatch, net, order, t, knobs):
    import paper_conf_ipps_maggionibl13_b200 as cme
    for k, v in knobs.items():
        monkeypatch.setenv(k, v)
    states, r, c, v = oracle_mod.enumerate_network(net)
    A = oracle_mod.ingest(len(states), r, c, v)
    m = cme.Matrix(A.n, r, c, v).reorder({"none": 0, "dfs": 1, "rcm": 2}[order]).pack()
    p, terms = m.transient(t)
    ref, rterms, lam = oracle_mod.transient(A, t)
    assert terms == rterms
    assert np.abs(p - ref).sum() <= 1e-12
    p0 = W.random_start(A.n, 5); p0 /= p0.sum()
    p, terms = m.transient(t, p0=p0)
    ref, _, _ = oracle_mod.transient(A, t, p0=p0)
    assert np.abs(p - ref).sum() <= 1e-12
    # the steady solve still works on the same handle afterwards
    m.set_opts(omega=0.9)
    _, st, _ = m.solve(tol=1e-10, max_iter=200000)
    assert st == "CONVERGED"


@pytest.mark.gpu
def test_gpu_transient_closed_form():
    import paper_conf_ipps_maggionibl13_b200 as cme
    m = cme.Matrix.from_network(W.birth_death(100, 10.0, 1.0)).pack()
    for t in (0.1, 1.0, 5.0):
        p, _ = m.transient(t)
        mm = 10.0 * (1.0 - math.exp(-t))
        ref = np.array([math.exp(-mm + x * math.log(mm) - math.lgamma(x + 1)) for x in range(101)])
        assert np.abs(p - ref).sum() < 1e-12
