"""Pins for the oracle's orderings, period test and packer.

* DFS: a hand-worked graph whose preorder is written out below; bijection.
* RCM: a shuffled path has bandwidth 1, a k x k grid bandwidth k; profile no
  worse than scipy's reverse_cuthill_mckee (sanity only, not bit-exact).
* period: cycles of length 2 and 3, and the networks' known periods.
* pack: unpack(pack(A)) == A bit for bit; ELL efficiency e = nnz/(n' k)
  (P:L135); the 2/3 band rule; rearrangement order.
"""
import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse.csgraph import reverse_cuthill_mckee

import workloads as W


def csr_from_edges(oracle_mod, n, edges, rate=1.0):
    """edges: (src j, dst i) transitions -> A_ij."""
    r = np.array([i for j, i in edges], np.int32)
    c = np.array([j for j, i in edges], np.int32)
    return oracle_mod.ingest(n, r, c, np.full(len(edges), rate))


def bandwidth(A, perm):
    inv = np.empty(A.n, np.int64); inv[perm] = np.arange(A.n)
    i = np.repeat(np.arange(A.n), np.diff(A.row_ptr))
    return int(np.abs(inv[i] - inv[A.col]).max()) if len(i) else 0


def test_dfs_hand_worked(oracle_mod):
    # transitions (j -> i); out-neighbours of 0 are {4, 1}, so ascending order
    # visits 1 first: 0,1,(1->3),3,(3->0 seen),(3->5),5,(5->4),4,(4->2),2,(2->0 seen)
    edges = [(0, 4), (0, 1), (1, 3), (3, 0), (3, 5), (5, 4), (4, 2), (2, 0), (2, 6), (6, 2)]
    A = csr_from_edges(oracle_mod, 7, edges)
    assert oracle_mod.order_dfs(A, 0).tolist() == [0, 1, 3, 5, 4, 2, 6]
    assert oracle_mod.order_dfs(A, 6).tolist() == [6, 2, 0, 1, 3, 5, 4]


def test_dfs_restarts_at_smallest_unvisited(oracle_mod):
    # two closed classes {0,1} and {2,3}; from root 3 the DFS covers {3,2} then restarts at 0
    A = csr_from_edges(oracle_mod, 4, [(0, 1), (1, 0), (2, 3), (3, 2)])
    assert oracle_mod.order_dfs(A, 3).tolist() == [3, 2, 0, 1]


# RCM hand-worked case (R12: George-Liu start, Cuthill-McKee by (degree, index),
# reverse).  Transitions j -> i; some edges one-way to exercise the A + A^T
# symmetrisation.  Undirected pattern and degrees:
#   0:{5,7} 2   1:{3,4} 2   2:{5,7} 2   3:{1,6,7,8} 4   4:{1,6} 2   5:{0,2} 2
#   6:{3,4} 2   7:{0,2,3} 3 8:{3} 1     9:{10} 1   10:{9,11} 2   11:{10} 1
# Component of 0 = {0..8}.  Start = min (degree, index) = 8.  BFS(8) levels
#   {8} {3} {1,6,7} {0,2,4} {5}: eccentricity 4; the last level's min is 5.
#   BFS(5): {5} {0,2} {7} {3} {1,6,8} {4}: eccentricity 5 > 4, so move to 5;
#   last level {4}; BFS(4): {4} {1,6} {3} {7,8} {0,2} {5}: 5, not > 5: stop.
# Cuthill-McKee from 5: 5 | nbrs 0,2 (deg 2, 2 -> by index) | from 0: 7 |
#   from 2: - | from 7: 3 | from 3: 8 (deg 1), 1, 6 (deg 2) | from 8: - |
#   from 1: 4 | -> [5,0,2,7,3,8,1,6,4].
# Component of 9 = {9,10,11}: start 9 (deg 1); BFS(9) eccentricity 2, last
#   level {11}, BFS(11) also 2: stay at 9 -> [9,10,11].
# Reverse of the concatenation: [11,10,9,4,6,1,8,3,7,2,0,5].
RCM_HAND_EDGES = [(5, 2), (2, 5), (0, 5), (2, 7), (7, 0), (7, 3), (3, 7), (1, 3), (3, 6), (6, 3), (4, 1),
                  (6, 4), (4, 6), (8, 3), (3, 8), (9, 10), (10, 11), (11, 10)]
RCM_HAND_PERM = [11, 10, 9, 4, 6, 1, 8, 3, 7, 2, 0, 5]


def test_rcm_hand_worked(oracle_mod):
    A = csr_from_edges(oracle_mod, 12, RCM_HAND_EDGES)
    assert oracle_mod.order_rcm(A).tolist() == RCM_HAND_PERM


def test_rcm_path_and_grid(oracle_mod):
    rng = np.random.default_rng(0)
    n = 200
    lab = rng.permutation(n)
    edges = []
    for a in range(n - 1):
        edges += [(lab[a], lab[a + 1]), (lab[a + 1], lab[a])]
    A = csr_from_edges(oracle_mod, n, edges)
    p = oracle_mod.order_rcm(A)
    assert sorted(p.tolist()) == list(range(n)) and bandwidth(A, p) == 1
    k = 12
    lab = rng.permutation(k * k)
    edges = []
    for r in range(k):
        for c in range(k):
            v = lab[r * k + c]
            if c + 1 < k:
                edges += [(v, lab[r * k + c + 1]), (lab[r * k + c + 1], v)]
            if r + 1 < k:
                edges += [(v, lab[(r + 1) * k + c]), (lab[(r + 1) * k + c], v)]
    G = csr_from_edges(oracle_mod, k * k, edges)
    assert bandwidth(G, oracle_mod.order_rcm(G)) == k


def test_rcm_vs_scipy_profile(oracle_mod):
    A = oracle_mod.network_csr(W.toggle_switch(60))
    i = np.repeat(np.arange(A.n), np.diff(A.row_ptr))
    S = sp.csr_matrix((np.ones(len(i)), (i, A.col)), shape=(A.n, A.n))
    S = ((S + S.T) > 0).astype(np.float64).tocsr()
    ps = reverse_cuthill_mckee(S, symmetric_mode=True)
    po = oracle_mod.order_rcm(A)
    assert sorted(po.tolist()) == list(range(A.n))
    assert bandwidth(A, po) <= 1.25 * bandwidth(A, ps)
    assert bandwidth(A, po) < bandwidth(A, np.arange(A.n)) / 4  # RCM beats DFS order


def test_permute_preserves_matrix(oracle_mod):
    A = oracle_mod.network_csr(W.schnakenberg(10))
    p = np.random.default_rng(1).permutation(A.n).astype(np.int32)
    B = oracle_mod.permute(A, p)
    Ad, Bd = A.dense(), B.dense()
    assert np.array_equal(Bd, Ad[np.ix_(p, p)])
    assert all(np.all(np.diff(B.col[B.row_ptr[r]:B.row_ptr[r + 1]]) > 0) for r in range(B.n))


def test_period_cycles_and_networks(oracle_mod):
    for L in (2, 3, 5):
        A = csr_from_edges(oracle_mod, L, [(a, (a + 1) % L) for a in range(L)])
        assert oracle_mod.period(A) == L
    # 2-cycle + 3-cycle sharing a vertex: gcd(2,3) = 1
    A = csr_from_edges(oracle_mod, 4, [(0, 1), (1, 0), (0, 2), (2, 3), (3, 0)])
    assert oracle_mod.period(A) == 1
    assert oracle_mod.period(oracle_mod.network_csr(W.toggle_switch(20))) == 2
    assert oracle_mod.period(oracle_mod.network_csr(W.brusselator(20))) == 2
    assert oracle_mod.period(oracle_mod.network_csr(W.schnakenberg(20))) == 1


def unpack(P, n):
    """Rebuild {(row, col): val} and inv_d[row] from layout v0 arrays."""
    ent, invd = {}, np.zeros(n)
    for s in range(P["n_slots"]):
        if s >= n:
            continue
        q, l = divmod(s, 32)
        r = int(P["row_of"][s])
        invd[r] = P["inv_d"][s]
        if P["band_on"]:
            if r >= 1 and P["lo"][s] != 0.0:
                ent[(r, r - 1)] = P["lo"][s]
            if r + 1 < n and P["up"][s] != 0.0:
                ent[(r, r + 1)] = P["up"][s]
        base = P["slice_off"][q] + l
        for t in range(P["slice_w"][q]):
            v, c = P["val"][base + 32 * t], P["col"][base + 32 * t]
            if v != 0.0:
                assert (r, c) not in ent
                ent[(r, int(c))] = v
            else:
                assert c == r
    return ent, invd


@pytest.mark.parametrize("window,band,uniform", [(256, "auto", False), (1, "auto", False),
                                                 (256, "never", False), (64, "always", False),
                                                 (1, "never", True)])
def test_pack_roundtrip(oracle_mod, window, band, uniform):
    for net in (W.toggle_switch(23), W.schnakenberg(19), W.birth_death(70)):
        A = oracle_mod.network_csr(net)
        P = oracle_mod.pack(A, window=window, band=band, uniform=uniform)
        ent, invd = unpack(P, A.n)
        ref = {}
        for i in range(A.n):
            for q in range(A.row_ptr[i], A.row_ptr[i + 1]):
                ref[(i, int(A.col[q]))] = A.val[q]
        assert ent == ref
        assert np.array_equal(invd, 1.0 / (-A.diag))
        assert sorted(P["row_of"][:A.n].tolist()) == list(range(A.n))
        assert P["n_slots"] % 32 == 0 and P["n_slots"] - A.n < 32
        assert np.all(P["slice_off"] % 32 == 0)
        if uniform:
            assert len(set(P["slice_w"].tolist())) == 1


def test_pack_rearrangement_and_efficiency(oracle_mod):
    A = oracle_mod.network_csr(W.toggle_switch(40))
    c = np.diff(A.row_ptr)
    for window in (1, 256):
        P = oracle_mod.pack(A, window=window, band="never")
        ro = P["row_of"][:A.n]
        for w0 in range(0, A.n, max(window, 1)):
            blk = ro[w0:w0 + window]
            assert sorted(blk.tolist()) == list(range(w0, min(w0 + window, A.n)))
            key = [(-c[r], r) for r in blk]
            assert key == sorted(key) or window == 1
        # slice width = exact max of its rows; e = nnz / stored slots
        for q in range(P["n_slices"]):
            rows = [r for r in P["row_of"][32 * q:32 * q + 32] if r < A.n]
            assert P["slice_w"][q] == max(c[rows])
        e = A.nnz_offdiag / P["n_ell"]
        if window == 1:
            e1 = e
    assert e >= e1   # local rearrangement never lowers the SELL efficiency here
    Pe = oracle_mod.pack(A, window=1, band="never", uniform=True)
    assert Pe["n_ell"] == Pe["n_slots"] * c.max()   # plain ELL: n' x k
    Pb = oracle_mod.pack(A, window=1, band="never", group=8)   # 256-row block slices [5]
    for g0 in range(0, Pb["n_slices"], 8):
        blk = list(range(32 * g0, min(32 * g0 + 256, A.n)))
        assert set(Pb["slice_w"][g0:g0 + 8]) == {max(c[blk])}
    Pw = oracle_mod.pack(A, window=1, band="never")
    assert Pw["n_ell"] <= Pb["n_ell"] <= Pe["n_ell"]   # warp-grained <= block-sliced <= ELL


def test_band_rule_threshold(oracle_mod):
    """DIA is on iff the +-1 density >= 2/3 = 8 B / 12 B."""
    n = 30

    def mat(n_band):  # ring with chords; first n_band sub-diagonal links are +-1 neighbours
        edges = set()
        for j in range(n):
            edges.add((j, (j + 7) % n)); edges.add(((j + 7) % n, j))
        pairs = 0
        for j in range(n - 1):
            if pairs < n_band:
                edges.add((j, j + 1)); edges.add((j + 1, j)); pairs += 1
        return csr_from_edges(oracle_mod, n, sorted(edges))

    for k in range(n):
        A = mat(k)
        i = np.repeat(np.arange(n), np.diff(A.row_ptr))
        cnt = int(((A.col == i - 1) | (A.col == i + 1)).sum())
        P = oracle_mod.pack(A)
        assert P["band_on"] == (3 * cnt >= 2 * (2 * n - 2))


@pytest.mark.parametrize("order", ["none", "rcm"])
@pytest.mark.parametrize("window,band", [(256, "auto"), (1, "never"), (64, "always")])
def test_compact_decodes_to_jacobi_matrix(oracle_mod, order, window, band):
    """Compact encoding pinned to the method, not to its own
    formula: decoding (row = window base + row8, col = row + col16) must give
    exactly the off-diagonal pattern of A; the decoded M applied to x must equal
    the oracle's C Jacobi step (divide last, eq. 8) within (k+2)u; and
    |d|^T M = |d|^T (the column-sum identity of the generator)."""
    net = W.toggle_switch(30)
    states, r, c, v = oracle_mod.enumerate_network(net)
    A0 = oracle_mod.ingest(len(states), r, c, v)
    A = A0 if order == "none" else oracle_mod.permute(A0, oracle_mod.order_rcm(A0))
    P = oracle_mod.pack(A, window=window, band=band)
    Q = oracle_mod.compact(A, P)
    assert Q is not None and Q["win_shift"] == (window.bit_length() - 1 if window > 1 else 0)
    n = A.n
    rows, cols, vals = [], [], []
    for s in range(n):
        q, lane = divmod(s, 32)
        rr = (s >> Q["win_shift"] << Q["win_shift"]) + int(Q["row8"][s]) if window > 1 else s
        for t in range(P["slice_w"][q]):
            e = P["slice_off"][q] + 32 * t + lane
            if Q["val"][e] != 0.0:
                rows.append(rr); cols.append(rr + int(Q["col16"][e])); vals.append(Q["val"][e])
        if P["band_on"]:
            for dj, key in ((-1, "lo"), (1, "up")):
                if Q[key][s] != 0.0:
                    rows.append(rr); cols.append(rr + dj); vals.append(Q[key][s])
    M = sp.csr_matrix((vals, (rows, cols)), shape=(n, n))
    ref = sp.csr_matrix((A.val, A.col, A.row_ptr), shape=(n, n))
    assert M.nnz == A.nnz_offdiag
    assert np.array_equal(M.indptr, ref.indptr) and np.array_equal(M.indices, ref.indices)
    x = np.random.default_rng(3).random(n)
    y_ref = oracle_mod.jacobi_step(A, x, omega=1.0)
    k = np.diff(A.row_ptr)
    assert np.all(np.abs(M @ x - y_ref) <= (k + 2) * 2.0 ** -53 * y_ref + 1e-300)
    dabs = -A.diag
    assert np.allclose(M.T @ dabs, dabs, rtol=1e-14, atol=0)


def test_compact_rejects_wide_offsets_and_windows(oracle_mod):
    """A transition spanning more than 32767 states, or a non-power-of-two
    window, has no compact encoding."""
    n = 40000
    edges = [(j, j + 1) for j in range(n - 1)] + [(j + 1, j) for j in range(n - 1)] + [(0, n - 1)]
    A = csr_from_edges(oracle_mod, n, edges)
    assert oracle_mod.compact(A, oracle_mod.pack(A, window=256)) is None
    B = csr_from_edges(oracle_mod, 100, [(j, j + 1) for j in range(99)] + [(j + 1, j) for j in range(99)])
    assert oracle_mod.compact(B, oracle_mod.pack(B, window=96)) is None
    assert oracle_mod.compact(B, oracle_mod.pack(B, window=128)) is not None


@pytest.mark.parametrize("net", [W.toggle_switch(40), W.schnakenberg(25), W.brusselator(30), W.birth_death(60)],
                         ids=lambda n: n.name)
@pytest.mark.parametrize("band", ["never", "always"])
def test_value_index_reconstructs_layout(oracle_mod, net, band):
    """Value-indexed form: dict[index] gives back every
    stored value of layout v0 bit for bit (val, and lo/up when the band is on),
    the dictionary is strictly ascending, and its size is the number of
    distinct stored values (mass-action rates: r_k times small integers)."""
    states, r, c, v = oracle_mod.enumerate_network(net)
    A = oracle_mod.ingest(len(states), r, c, v)
    P = oracle_mod.pack(A, window=256, band=band)
    V = oracle_mod.value_index(P)
    assert V is not None
    d = V["dict"]
    assert np.all(np.diff(d) > 0)
    assert d[V["vidx"]].tobytes() == P["val"].tobytes()
    if P["band_on"]:
        assert d[V["loi"]].tobytes() == P["lo"].tobytes() and d[V["upi"]].tobytes() == P["up"].tobytes()
    stored = set(P["val"].tolist()) | (set(P["lo"].tolist()) | set(P["up"].tolist()) if P["band_on"] else set())
    assert len(d) == len(stored)
    assert len(d) <= len(np.unique(v)) + 1       # + the pad value 0.0


def test_value_index_limit(oracle_mod):
    """More than 65536 distinct values: no value-indexed form."""
    n = 70000
    r, c, v = W.banded_markov(n, 5, 64, False, seed=2)
    A = oracle_mod.ingest(n, r, c, v)
    assert oracle_mod.value_index(oracle_mod.pack(A, window=256)) is None
