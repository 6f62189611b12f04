"""Pins for the oracle's Jacobi iteration and dense LU.

Closed forms (textbook, not the oracle's formulas):
* birth-death truncated Poisson  pi_x ~ (lam/mu)^x / x!;
* Schnakenberg under detailed balance: product Poisson a^x b^y / (x! y!)
  on the triangle x + y <= N;
* Schloegl (1-D): pi_x ~ prod_{y<=x} birth(y-1)/death(y);
* closed cyclic A->B->C->A with linear rates: pi ~ 1/(a! b! c!);
plus numpy.linalg.solve (LAPACK dgesv), dense numpy products, and invariants.
"""
import math
import os

import numpy as np
import pytest

import workloads as W


def poisson_trunc(lam, N):
    logs = np.array([x * math.log(lam) - math.lgamma(x + 1) for x in range(N + 1)])
    p = np.exp(logs - logs.max())
    return p / p.sum()


def product_poisson(states, a, b):
    logs = np.array([x * math.log(a) - math.lgamma(x + 1) + y * math.log(b) - math.lgamma(y + 1)
                     for x, y in states])
    p = np.exp(logs - logs.max())
    return p / p.sum()


@pytest.fixture(scope="module")
def bd(oracle_mod):
    return oracle_mod.network_csr(W.birth_death(100, 10.0, 1.0))


def test_lu_birth_death_closed_form(oracle_mod, bd):
    p = oracle_mod.lu_steady(bd)
    assert np.abs(p - poisson_trunc(10.0, 100)).sum() < 1e-13


def test_lu_matches_lapack(oracle_mod):
    for net in (W.toggle_switch(10), W.cyclic3(5), W.schnakenberg(12, 8, 1, 5, 1, 0.01)):
        A = oracle_mod.network_csr(net)
        M = A.dense()
        M[-1, :] = 1.0
        e = np.zeros(A.n); e[-1] = 1.0
        ref = np.linalg.solve(M, e)
        assert np.abs(oracle_mod.lu_steady(A) - ref).sum() < 1e-12


def test_jacobi_birth_death_damped(oracle_mod, bd):
    r = oracle_mod.jacobi_solve(bd, omega=0.9, tol=1e-14, max_iter=200000)
    assert r.status == "CONVERGED" and r.iters % 100 == 0
    assert np.abs(r.p - poisson_trunc(10.0, 100)).sum() < 1e-11


@pytest.mark.parametrize("omega", [0.9, 0.3, 1.0])
def test_damping_on_the_minus_one_eigenvector(oracle_mod, bd, omega):
    """Where omega sits in the damped step (R1), pinned by the spectrum, not by
    restating the formula.  A u = 0 <=> O u = |D| u <=> M u = u for
    M = |D|^-1 O, and u = the truncated Poisson law (closed form).  The
    birth-death chain is bipartite: O only links x to x +- 1, so with
    S = diag((-1)^x), O S = -S O and M (S u) = -S u.  Hence
    M_omega (S u) = (1 - 2 omega) S u; a swapped omega <-> 1 - omega would
    give 2 omega - 1 instead (+0.8 vs -0.8 at omega = 0.9)."""
    u = poisson_trunc(10.0, 100)             # A u = 0  <=>  M u = u (M = |D|^-1 O)
    S = np.where(np.arange(101) % 2 == 0, 1.0, -1.0)
    v = S * u
    y = oracle_mod.jacobi_step(bd, v, omega)
    ref = (1.0 - 2.0 * omega) * v
    big = np.abs(v) > 1e-200
    assert np.max(np.abs(y[big] - ref[big]) / np.abs(v[big])) < 1e-12


@pytest.mark.slow
@pytest.mark.parametrize("omega,status,iters", [(0.9, "CONVERGED", 3400), (0.5, "CONVERGED", 5900),
                                                (1.0, "STAGNATED", None)])
def test_survey_c3_toggle_iteration_counts(oracle_mod, omega, status, iters):
    """SURVEY C3 / F2 (an independent computation, recorded at survey time):
    config 2 (toggle switch N = 224, 99 908 states), uniform p0, C = 100,
    tol 1e-12: omega = 0.9 stops at 3 400 iterations, omega = 0.5 at 5 900, and
    pure Jacobi (omega = 1) stalls with delta = 1.404e-5 (period 2)."""
    A = oracle_mod.network_csr(W.toggle_switch(224))
    assert A.n == 99908
    r = oracle_mod.jacobi_solve(A, omega=omega, tol=1e-12, max_iter=20000, nthreads=os.cpu_count() or 1)
    assert r.status == status
    if iters is not None:
        assert r.iters == iters and r.delta <= 1e-12
    else:
        assert r.delta == pytest.approx(1.404e-5, rel=1e-3)


def test_pure_jacobi_stagnates_on_period_two(oracle_mod, bd):
    """omega = 1 on a bipartite chain oscillates (eigenvalue -1)."""
    assert oracle_mod.period(bd) == 2
    r = oracle_mod.jacobi_solve(bd, omega=1.0, tol=1e-14, max_iter=200000)
    assert r.status == "STAGNATED"
    assert r.delta > 1e-6


def test_cyclic_period_three(oracle_mod):
    A = oracle_mod.network_csr(W.cyclic3(3))
    assert oracle_mod.period(A) == 3
    assert oracle_mod.jacobi_solve(A, omega=1.0, tol=1e-14, max_iter=100000).status == "STAGNATED"
    states, *_ = oracle_mod.enumerate_network(W.cyclic3(3))
    pi = np.array([1.0 / (math.factorial(a) * math.factorial(b) * math.factorial(c)) for a, b, c in states])
    pi /= pi.sum()
    r = oracle_mod.jacobi_solve(A, omega=0.9, tol=1e-15, max_iter=100000)
    assert r.status == "CONVERGED" and np.abs(r.p - pi).sum() < 1e-13


def test_schnakenberg_detailed_balance(oracle_mod):
    net = W.schnakenberg(40, 8.0, 1.0, 5.0, 1.0, 0.01)
    states, r_, c_, v_ = oracle_mod.enumerate_network(net)
    A = oracle_mod.ingest(len(states), r_, c_, v_)
    pi = product_poisson(states, 8.0, 5.0)
    assert np.abs(oracle_mod.lu_steady(A) - pi).sum() < 1e-13
    assert oracle_mod.period(A) == 1
    r = oracle_mod.jacobi_solve(A, omega=1.0, tol=1e-15, max_iter=100000)
    assert r.status == "CONVERGED"
    assert np.abs(r.p - pi).sum() < 1e-12


def test_schlogl_closed_form(oracle_mod):
    net = W.schlogl(700)
    c1, c2, c3, c4 = (net.meta[k] for k in ("c1", "c2", "c3", "c4"))
    A = oracle_mod.network_csr(net)
    logs = [0.0]
    for y in range(1, 701):
        birth = c1 * math.comb(y - 1, 2) + c3
        death = c2 * math.comb(y, 3) + c4 * y
        logs.append(logs[-1] + math.log(birth) - math.log(death))
    logs = np.array(logs)
    pi = np.exp(logs - logs.max()); pi /= pi.sum()
    p = oracle_mod.lu_steady(A)
    assert np.abs(p - pi).sum() < 1e-12
    modes = [i for i in range(1, 700) if pi[i] > pi[i - 1] and pi[i] > pi[i + 1]]
    assert modes == [96, 389]     # bistable


@pytest.mark.parametrize("omega", [1.0, 0.9, 0.5])
def test_step_matches_dense(oracle_mod, omega):
    """y = (1-w) x + w |D|^{-1} (L+U) x, with numpy's dense product."""
    A = oracle_mod.network_csr(W.toggle_switch(9))
    M = A.dense()
    D = np.diag(M).copy()
    O = M - np.diag(D)
    x = W.random_start(A.n, 3)
    ref = (1 - omega) * x + omega * (O @ x) / (-D)
    y = oracle_mod.jacobi_step(A, x, omega)
    assert np.max(np.abs(y - ref) / ref) < 1e-14


def test_unnormalised_step_conserves_weighted_mass(oracle_mod):
    """|d|^T is a left eigenvector of M_omega with eigenvalue 1."""
    A = oracle_mod.network_csr(W.toggle_switch(30))
    x = W.random_start(A.n, 1)
    d = -A.diag
    m0 = (d * x).sum()
    for omega in (1.0, 0.7):
        y = x
        for _ in range(20):
            y = oracle_mod.jacobi_step(A, y, omega)
        assert abs((d * y).sum() - m0) <= 1e-13 * m0
    assert np.all(y >= 0)


def test_paper_residual_definition(oracle_mod):
    """resid at the first check equals ||A x0||_inf / (||A||_inf ||x0||_inf)."""
    A = oracle_mod.network_csr(W.schnakenberg(15, 8, 1, 5, 1, 0.01))
    M = A.dense()
    x0 = W.random_start(A.n, 5); x0 /= x0.sum()
    for omega in (1.0, 0.8):
        r = oracle_mod.jacobi_solve(A, p0=x0, omega=omega, tol=0.0, check_every=1, max_iter=1)
        ref = np.abs(M @ x0).max() / (np.abs(M).sum(axis=1).max() * x0.max())
        assert r.resid == pytest.approx(ref, rel=1e-12)
        y = (1 - omega) * x0 + omega * ((M - np.diag(np.diag(M))) @ x0) / (-np.diag(M))
        assert r.delta == pytest.approx(np.abs(y - x0).sum(), rel=1e-12)


def test_threads_bit_identical(oracle_mod):
    A = oracle_mod.network_csr(W.toggle_switch(60))
    a = oracle_mod.jacobi_solve(A, omega=0.9, tol=1e-12, max_iter=3000, nthreads=1)
    b = oracle_mod.jacobi_solve(A, omega=0.9, tol=1e-12, max_iter=3000, nthreads=4)
    assert a.iters == b.iters and np.array_equal(a.p, b.p)


def test_max_iter_and_partial_block(oracle_mod, bd):
    r = oracle_mod.jacobi_solve(bd, omega=0.9, tol=0.0, max_iter=250)
    assert r.status == "NOT_CONVERGED" and r.iters == 250
    assert r.p.sum() == pytest.approx(1.0, abs=1e-14)
    r0 = oracle_mod.jacobi_solve(bd, omega=0.9, tol=0.0, max_iter=0)
    assert r0.iters == 0 and np.allclose(r0.p, 1.0 / bd.n)


def test_toggle_landscape_bimodal(oracle_mod):
    """Fig. 2 / P:L79: mass concentrates on on/off and off/on."""
    states, r_, c_, v_ = oracle_mod.enumerate_network(W.toggle_switch(80))
    A = oracle_mod.ingest(len(states), r_, c_, v_)
    r = oracle_mod.jacobi_solve(A, omega=0.9, tol=1e-12, max_iter=100000)
    assert r.status == "CONVERGED"
    pA, pB = states[:, 0], states[:, 1]
    onoff = r.p[(pA >= 20) & (pB < 5)].sum()
    offon = r.p[(pB >= 20) & (pA < 5)].sum()
    assert onoff > 0.35 and offon > 0.35 and abs(onoff - offon) < 1e-6
