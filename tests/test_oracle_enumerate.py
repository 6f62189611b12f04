"""Pins for the oracle's enumerator + ingest (Table I).

Everything here is `not gpu`.  Pins are independent of the oracle's own code:
Table I values printed in the paper (tests/golden/table1.txt), closed-form
state counts, a brute-force Python breadth-first enumeration with math.comb
propensities, and exact zero column sums.
"""
import math
import os

import numpy as np
import pytest

import workloads as W

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "table1.txt")


def T(k):
    return (k + 1) * (k + 2) // 2 if k >= 0 else 0


def row_stats(A):
    nnz_row = np.diff(A.row_ptr) + 1  # + diagonal (Table I counts it)
    mu = nnz_row.mean()
    i = np.repeat(np.arange(A.n), np.diff(A.row_ptr))
    band = int(((A.col == i - 1) | (A.col == i + 1)).sum())
    return dict(n=A.n, nnz=A.nnz, min=int(nnz_row.min()), mu=mu, max=int(nnz_row.max()),
                sigma=nnz_row.std(), cv=nnz_row.std() / mu, skew=(nnz_row.max() - mu) / mu,
                d0=1.0, d1=(band + A.n) / (3 * A.n - 2))


def golden_rows():
    rows = []
    for line in open(GOLDEN):
        if line.startswith("#") or not line.strip():
            continue
        f = line.split()
        rows.append(dict(name=f[0], N=int(f[1]), n=int(f[2]), nnz=int(f[3]), min=int(f[4]),
                         mu=float(f[5]), max=int(f[6]), sigma=float(f[7]), cv=float(f[8]),
                         skew=float(f[9]), d0=float(f[10]), d1=float(f[11])))
    return rows


NETS = {"toggle_switch": W.toggle_switch, "brusselator": W.brusselator,
        "schnakenberg": W.schnakenberg}


@pytest.mark.slow
@pytest.mark.parametrize("row", golden_rows(), ids=lambda r: r["name"])
def test_table1_row_reproduced(oracle_mod, row):
    """Every Table I column of the three reproducible networks."""
    A = oracle_mod.network_csr(NETS[row["name"]](row["N"]))
    s = row_stats(A)
    assert s["n"] == row["n"] and s["nnz"] == row["nnz"]
    assert s["min"] == row["min"] and s["max"] == row["max"]
    for key in ("mu", "sigma", "cv", "skew", "d0"):
        assert round(s[key], 2) == pytest.approx(row[key], abs=1e-9), key
    if row["name"] != "toggle_switch":  # reaction order of [17] unknown
        assert round(s["d1"], 2) == pytest.approx(row["d1"], abs=1e-9)
    else:
        assert abs(s["d1"] - row["d1"]) < 0.05


@pytest.mark.parametrize("N", [3, 4, 7, 20, 41])
def test_state_count_closed_forms(oracle_mod, N):
    """n(N), nnz(N) by counting:
    toggle: gene states (GAb,GBb) in {0,1}^2 leave pA+pB <= N-2(GAb+GBb):
    n = T(N)+2T(N-2)+T(N-4) = 2N^2-2N+4 (N >= 4); schnakenberg n = T(N);
    brusselator n = T(N)-1 (the zero-outflow corner (0,N) is deleted)."""
    tog = oracle_mod.network_csr(W.toggle_switch(N))
    assert tog.n == T(N) + 2 * T(N - 2) + T(N - 4)
    if N >= 4:
        assert tog.n == 2 * N * N - 2 * N + 4 and tog.nnz == 12 * N * N - 28 * N + 34
    sch = oracle_mod.network_csr(W.schnakenberg(N))
    assert sch.n == T(N) and sch.nnz == T(N) + 4 * T(N - 1) + 2 * T(N - 3)
    bru = oracle_mod.network_csr(W.brusselator(N))
    assert bru.n == T(N) - 1
    assert bru.nnz == T(N) + 3 * T(N - 1) + T(N - 3) - 2


def brute_force(net):
    """Independent breadth-first enumeration with math.comb propensities:
    returns {state: {target: rate}} for the states that survive zero-outflow pruning."""
    x0, reac, chg, rates, w, cap = net.arrays()
    start = tuple(int(v) for v in x0)
    seen = {start}
    frontier = [start]
    edges = {}
    while frontier:
        nxt = []
        for x in frontier:
            out = {}
            for k in range(net.R):
                prod = 1
                for i in range(net.m):
                    prod *= math.comb(x[i], int(reac[k, i])) if x[i] >= reac[k, i] else 0
                a = float(rates[k]) * float(prod)
                y = tuple(x[i] + int(chg[k, i]) for i in range(net.m))
                if a <= 0 or min(y) < 0 or sum(int(w[i]) * y[i] for i in range(net.m)) > cap:
                    continue
                out[y] = out.get(y, 0.0) + a
                if y not in seen:
                    seen.add(y)
                    nxt.append(y)
            edges[x] = out
        frontier = nxt
    alive = set(edges)
    changed = True
    while changed:
        changed = False
        for x in list(alive):
            if not any(y in alive for y in edges[x]):
                alive.discard(x)
                changed = True
    return {x: {y: r for y, r in edges[x].items() if y in alive} for x in alive}


@pytest.mark.parametrize("net", [W.toggle_switch(6), W.brusselator(6), W.schnakenberg(6),
                                 W.birth_death(9), W.schlogl(12), W.cyclic3(4)],
                         ids=lambda n: n.name)
def test_bruteforce_small(oracle_mod, net):
    states, r, c, v = oracle_mod.enumerate_network(net)
    bf = brute_force(net)
    got = [tuple(s) for s in states]
    assert set(got) == set(bf) and len(got) == len(bf)
    assert got[0] == tuple(net.x0)
    A = oracle_mod.ingest(len(states), r, c, v)
    for j, xj in enumerate(got):
        for i_, rate in bf[xj].items():
            i = got.index(i_)
            row = A.col[A.row_ptr[i]:A.row_ptr[i + 1]]
            assert j in row
            assert A.val[A.row_ptr[i] + int(np.nonzero(row == j)[0][0])] == rate
        assert -A.diag[j] == pytest.approx(sum(bf[xj].values()), rel=1e-15)


def is_dfs_preorder(states, net):
    """Check the DEFINING property of a DFS preorder over the reaction graph
    (children tried in reaction order): replaying the order with a stack, every
    next state must be an unvisited successor of the deepest state on the stack
    that still has one, and it must be that state's FIRST such successor."""
    x0, reac, chg, rates, w, cap = net.arrays()
    bf = brute_force(net)
    index = {tuple(s): i for i, s in enumerate(states)}

    def succ(x):  # reaction-ordered successors of x (with duplicates removed)
        out = []
        for k in range(net.R):
            y = tuple(x[i] + int(chg[k, i]) for i in range(net.m))
            if y in bf.get(x, {}) and y not in out:
                out.append(y)
        return out

    visited = {tuple(states[0])}
    stack = [tuple(states[0])]
    for s in states[1:]:
        s = tuple(s)
        while stack:
            cand = [y for y in succ(stack[-1]) if y not in visited]
            if cand:
                break
            stack.pop()
        if not stack or cand[0] != s:
            return False
        visited.add(s)
        stack.append(s)
    return len(visited) == len(index)


@pytest.mark.parametrize("net", [W.schnakenberg(5), W.birth_death(7), W.cyclic3(3)],
                         ids=lambda n: n.name)
def test_enumeration_is_dfs_preorder(oracle_mod, net):
    # (networks with no zero-outflow pruning, so preorder positions are untouched)
    states, *_ = oracle_mod.enumerate_network(net)
    assert is_dfs_preorder(states, net)


def test_zero_column_sums_exact(oracle_mod):
    """A(x,x) = -sum_{x' != x} A(x',x): with integer rates every partial
    sum is an exact integer, so column sums of A vanish exactly."""
    A = oracle_mod.network_csr(W.brusselator(60))
    colsum = np.zeros(A.n)
    np.add.at(colsum, A.col, A.val)
    assert np.all(colsum + A.diag == 0.0)
    assert np.all(A.diag < 0) and np.all(A.val > 0)


def test_brusselator_corner_pruned(oracle_mod):
    states, *_ = oracle_mod.enumerate_network(W.brusselator(10))
    assert (0, 10) not in {tuple(s) for s in states}
    assert len(states) == T(10) - 1


def test_ingest_duplicates_summed_in_input_order(oracle_mod):
    r = np.array([1, 1, 1, 0, 2, 0], np.int32)
    c = np.array([0, 0, 0, 1, 1, 2], np.int32)
    v = np.array([0.1, 0.2, 0.3, 1.0, 2.0, 5.0])
    A = oracle_mod.ingest(3, r, c, v)
    assert A.row_ptr.tolist() == [0, 2, 3, 4]
    assert A.col.tolist() == [1, 2, 0, 1]
    assert A.val[2] == (0.1 + 0.2) + 0.3
    assert A.diag.tolist() == [-((0.1 + 0.2) + 0.3), -3.0, -5.0]


def test_ingest_errors(oracle_mod):
    E = oracle_mod.OracleError
    with pytest.raises(E) as e:
        oracle_mod.ingest(2, [0], [1], [-1.0])
    assert e.value.code == 2
    with pytest.raises(E) as e:
        oracle_mod.ingest(2, [0, 1], [1, 0], [float("nan"), 1.0])
    assert e.value.code == 1
    with pytest.raises(E) as e:
        oracle_mod.ingest(2, [0, 1, 1], [1, 0, 1], [1.0, 1.0, 1.0])
    assert e.value.code == 1  # diagonal entry without CME_DIAG_GIVEN
    with pytest.raises(E) as e:
        oracle_mod.ingest(3, [0, 1], [1, 0], [1.0, 1.0])
    assert e.value.code == 3  # state 2 has no outflow
    with pytest.raises(E) as e:
        oracle_mod.ingest(2, [0, 5], [1, 0], [1.0, 1.0])
    assert e.value.code == 1


def test_ingest_diag_given(oracle_mod):
    A = oracle_mod.ingest(2, [0, 1, 0, 1], [1, 0, 0, 1], [2.0, 3.0, -3.0, -2.0], diag_given=True)
    assert A.diag.tolist() == [-3.0, -2.0] and A.val.tolist() == [2.0, 3.0]
    with pytest.raises(oracle_mod.OracleError):
        oracle_mod.ingest(2, [0, 1, 0, 1], [1, 0, 0, 1], [2.0, 3.0, -3.5, -2.0], diag_given=True)
