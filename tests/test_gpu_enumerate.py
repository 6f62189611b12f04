"""GPU state enumerator (cme_network_enumerate_gpu) against
the oracle's enumerator (eq. 1, readings R7-R10).

The GPU numbers states lexicographically instead of by DFS preorder, so the
oracle's output is mapped through the lexicographic permutation first; then
states, row/col indices and the rate bytes must match exactly (integer work
bit-exact; the rates are the same exact binomial products and one fp64
multiply).  Error paths run without a GPU.
"""
import numpy as np
import pytest

import workloads as W


@pytest.fixture(scope="module")
def cme():
    import paper_conf_ipps_maggionibl13_b200 as m
    return m


def lex_canonical(states, r, c, v):
    """Oracle enumeration -> lexicographic state numbering, triplets grouped by
    source state in their emission (reaction) order."""
    n, m = states.shape
    perm = np.lexsort(tuple(states[:, i] for i in range(m - 1, -1, -1)))   # new -> old
    inv = np.empty(n, dtype=np.int64)
    inv[perm] = np.arange(n)
    rr, cc = inv[r].astype(np.int32), inv[c].astype(np.int32)
    order = np.argsort(cc, kind="stable")
    return states[perm], rr[order], cc[order], v[order]


NETS = [W.toggle_switch(23), W.toggle_switch(60), W.brusselator(40), W.schnakenberg(35),
        W.birth_death(100), W.schlogl(200), W.cyclic3(5), W.brusselator(3)]


@pytest.mark.gpu
@pytest.mark.parametrize("net", NETS, ids=lambda n: n.name)
def test_gpu_enumeration_matches_oracle(cme, oracle_mod, net):
    ref = lex_canonical(*oracle_mod.enumerate_network(net))
    got = cme.cme_network_enumerate_gpu(net)
    for x, y in zip(ref, got):
        assert x.dtype == y.dtype and x.shape == y.shape and np.array_equal(x, y)
        if x.dtype == np.float64:
            assert x.tobytes() == y.tobytes()


@pytest.mark.gpu
def test_gpu_enumeration_solve_matches_dfs_enumeration(cme, oracle_mod):
    """A matrix built from the GPU enumeration solves to the same landscape
    (state by state) as the oracle's DFS-ordered one."""
    net = W.toggle_switch(40)
    st_o, r, c, v = oracle_mod.enumerate_network(net)
    A = oracle_mod.ingest(len(st_o), r, c, v)
    ref = oracle_mod.jacobi_solve(A, omega=0.9, tol=1e-12)
    m = cme.Matrix.from_network(net, gpu=True).reorder(cme.CME_ORDER_RCM).pack()
    m.set_opts(omega=0.9)
    p, st, it = m.solve(tol=1e-12)
    assert st == "CONVERGED"
    key = {tuple(s): i for i, s in enumerate(st_o)}
    idx = np.array([key[tuple(s)] for s in m.states])
    assert np.abs(p - ref.p[idx]).sum() <= 1e-10


@pytest.mark.gpu
@pytest.mark.slow
def test_gpu_enumeration_cfg4_full_size(cme, oracle_mod):
    """configs[3] (toggle N = 3164, n = 20,015,468): same states and triplets
    as the oracle's enumerator."""
    import time
    net = W.config_network("cfg4_toggle_20m")
    t = time.perf_counter()
    got = cme.cme_network_enumerate_gpu(net)
    t_gpu = time.perf_counter() - t
    ref = lex_canonical(*oracle_mod.enumerate_network(net))
    assert len(got[0]) == 20015468 and len(got[1]) == 120042194 - 20015468
    for x, y in zip(ref, got):
        assert np.array_equal(x, y)
    print(f"gpu enumeration of {len(got[0])} states: {t_gpu:.2f} s")


def test_gpu_enumerator_rejects_out_of_range(cme):
    """Counts beyond the 16-bit key fields are refused up front (x0) or during
    the BFS (without a GPU the call reports CME_ERR_NO_DEVICE first)."""
    import torch
    bad = W.Network(name="big_x0", species=["X"], x0=[70000], reactants=[[0], [1]], change=[[1], [-1]],
                    rates=[1.0, 1.0], weights=[1], cap=80000)
    with pytest.raises(cme.CmeError) as e:
        cme.cme_network_enumerate_gpu(bad)
    assert e.value.status == cme.CME_ERR_INVALID_ARG
    deep = W.birth_death(70000)
    with pytest.raises(cme.CmeError) as e:
        cme.cme_network_enumerate_gpu(deep)
    want = cme.CME_ERR_INVALID_ARG if torch.cuda.is_available() else cme.CME_ERR_NO_DEVICE
    assert e.value.status == want
