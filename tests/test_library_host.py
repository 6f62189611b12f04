"""Host-side parity of libcme against the oracle (no GPU needed).

Integer / byte work must match bit for bit (north star): enumeration, ingest,
orderings, the period test and the packed layout.  Also: the C-ABI library
loads and exports every symbol include/cme.h declares, and every error path
returns the documented status.
"""
import os
import re

import numpy as np
import pytest

import paper_conf_ipps_maggionibl13_b200 as cme
import workloads as W

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

NETS = [W.toggle_switch(23), W.toggle_switch(60), W.brusselator(40), W.schnakenberg(35),
        W.birth_death(100), W.schlogl(200), W.cyclic3(5)]


def header_functions():
    src = open(os.path.join(ROOT, "include", "cme.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(cme_[a-z0-9_]+)\s*\(", src)))


def test_abi_exports_every_declared_symbol():
    declared = header_functions()
    assert len(declared) >= 25
    for name in declared:
        assert hasattr(cme._lib, name), name
    assert sorted(declared) == cme.ABI_SYMBOLS
    assert cme.cme_abi_version() == 1
    assert cme.cme_status_string(cme.CME_STAGNATED) == "CME_STAGNATED"
    assert cme.cme_status_string(cme.CME_ERR_TIMEOUT) == "CME_ERR_TIMEOUT"


@pytest.mark.parametrize("net", NETS, ids=lambda n: n.name)
def test_enumeration_bit_exact(oracle_mod, net):
    a = oracle_mod.enumerate_network(net)
    b = cme.cme_network_enumerate(net)
    for x, y in zip(a, b):
        assert x.dtype == y.dtype and np.array_equal(x, y)
        if x.dtype == np.float64:
            assert x.tobytes() == y.tobytes()


def host_matrix(n, r, c, v, order=cme.CME_ORDER_NONE, root=0, fmt=cme.CME_FMT_DIAG_SELL, window=256,
                band=cme.CME_BAND_AUTO):
    m = cme.Matrix(n, r, c, v)
    m.reorder(order, root)
    m.pack(fmt, window, band, device=cme.CME_DEVICE_HOST_ONLY)
    return m


@pytest.mark.parametrize("net", NETS, ids=lambda n: n.name)
def test_ingest_bit_exact(oracle_mod, net):
    states, r, c, v = oracle_mod.enumerate_network(net)
    A = oracle_mod.ingest(len(states), r, c, v)
    m = host_matrix(len(states), r, c, v, fmt=cme.CME_FMT_CSR)
    P = m.packed()
    assert np.array_equal(P["csr_row_ptr"], A.row_ptr)
    assert np.array_equal(P["col"], A.col)
    assert P["val"].tobytes() == A.val.tobytes()
    assert P["inv_d"][:A.n].tobytes() == (1.0 / (-A.diag)).tobytes()
    f = m.info()
    assert f.n == A.n and f.nnz == A.nnz
    assert f.period == oracle_mod.period(A)


def test_ingest_duplicates_and_random_coo(oracle_mod):
    rng = np.random.default_rng(7)
    n, nnz = 300, 4000
    r = rng.integers(0, n, nnz).astype(np.int32)
    c = rng.integers(0, n, nnz).astype(np.int32)
    keep = r != c
    r, c = r[keep], c[keep]
    v = rng.random(len(r)) * 10.0 ** rng.integers(-3, 4, len(r))
    # make every column have outflow
    r = np.concatenate([r, (np.arange(n) + 1) % n]).astype(np.int32)
    c = np.concatenate([c, np.arange(n)]).astype(np.int32)
    v = np.concatenate([v, np.full(n, 0.5)])
    A = oracle_mod.ingest(n, r, c, v)
    P = host_matrix(n, r, c, v, fmt=cme.CME_FMT_CSR).packed()
    assert np.array_equal(P["csr_row_ptr"], A.row_ptr) and np.array_equal(P["col"], A.col)
    assert P["val"].tobytes() == A.val.tobytes()
    assert P["inv_d"][:n].tobytes() == (1.0 / (-A.diag)).tobytes()


@pytest.mark.parametrize("net", NETS, ids=lambda n: n.name)
@pytest.mark.parametrize("order", ["dfs", "rcm"])
def test_orderings_bit_exact(oracle_mod, net, order):
    states, r, c, v = oracle_mod.enumerate_network(net)
    A = oracle_mod.ingest(len(states), r, c, v)
    m = cme.Matrix(len(states), r, c, v)
    if order == "dfs":
        root = len(states) // 3
        m.reorder(cme.CME_ORDER_DFS, root)
        ref = oracle_mod.order_dfs(A, root)
    else:
        m.reorder(cme.CME_ORDER_RCM)
        ref = oracle_mod.order_rcm(A)
    assert np.array_equal(m.permutation(), ref)


def test_rcm_hand_worked_library():
    """cme_reorder(RCM) on the hand-worked graph of test_oracle_order_pack.py (R12)."""
    from test_oracle_order_pack import RCM_HAND_EDGES, RCM_HAND_PERM
    r = np.array([i for j, i in RCM_HAND_EDGES], np.int32)
    c = np.array([j for j, i in RCM_HAND_EDGES], np.int32)
    m = cme.Matrix(12, r, c, np.ones(len(r)))
    m.reorder(cme.CME_ORDER_RCM)
    assert m.permutation().tolist() == RCM_HAND_PERM


PACK_CASES = [("none", 256, "auto", cme.CME_FMT_DIAG_SELL), ("dfs", 256, "auto", cme.CME_FMT_DIAG_SELL),
              ("none", 1, "auto", cme.CME_FMT_SELL256), ("rcm", 1, "never", cme.CME_FMT_SELL256),
              ("rcm", 1 << 30, "never", cme.CME_FMT_DIAG_SELL),
              ("rcm", 256, "auto", cme.CME_FMT_DIAG_SELL), ("none", 1, "never", cme.CME_FMT_DIAG_SELL),
              ("rcm", 64, "always", cme.CME_FMT_DIAG_SELL), ("none", 1, "auto", cme.CME_FMT_ELL),
              ("dfs", 1, "never", cme.CME_FMT_ELL)]


@pytest.mark.parametrize("net", NETS, ids=lambda n: n.name)
@pytest.mark.parametrize("order,window,band,fmt", PACK_CASES)
def test_pack_bit_exact(oracle_mod, net, order, window, band, fmt):
    states, r, c, v = oracle_mod.enumerate_network(net)
    A = oracle_mod.ingest(len(states), r, c, v)
    om = {"none": cme.CME_ORDER_NONE, "dfs": cme.CME_ORDER_DFS, "rcm": cme.CME_ORDER_RCM}[order]
    bm = {"auto": cme.CME_BAND_AUTO, "always": cme.CME_BAND_ALWAYS, "never": cme.CME_BAND_NEVER}[band]
    m = host_matrix(len(states), r, c, v, om, 0, fmt, window, bm)
    perm = {"none": np.arange(A.n, dtype=np.int32), "dfs": oracle_mod.order_dfs(A, 0),
            "rcm": oracle_mod.order_rcm(A)}[order]
    ref = oracle_mod.pack(oracle_mod.permute(A, perm), window=window if fmt == cme.CME_FMT_DIAG_SELL else 1,
                          band=band, uniform=fmt == cme.CME_FMT_ELL,
                          group=8 if fmt == cme.CME_FMT_SELL256 else 1)
    got = m.packed()
    for key in ("n", "n_slots", "n_slices", "n_ell", "band_on", "window"):
        assert got[key] == ref[key], key
    for key in ("lo", "up", "inv_d", "row_of", "slice_off", "slice_w", "val", "col"):
        assert got[key].dtype == ref[key].dtype and got[key].tobytes() == ref[key].tobytes(), key
    # compact encoding: bit-exact too, or rejected by both
    refc = oracle_mod.compact(oracle_mod.permute(A, perm), ref)
    if refc is None:
        with pytest.raises(cme.CmeError):
            m.compact()
    else:
        gotc = m.compact()
        assert gotc["win_shift"] == refc["win_shift"]
        refv = oracle_mod.value_index(ref)   # value-indexed form (sec. 5c), when <= 65536 values
        if refv is not None:
            refc.update(refv)
        assert set(gotc) == set(refc)
        for key in refc:
            if key != "win_shift":
                assert gotc[key].dtype == refc[key].dtype and gotc[key].tobytes() == refc[key].tobytes(), key


def test_given_permutation_bit_exact(oracle_mod):
    """A seeded random ordering (the locality stress test of P:L225) passed to both sides."""
    states, r, c, v = oracle_mod.enumerate_network(W.toggle_switch(40))
    A = oracle_mod.ingest(len(states), r, c, v)
    perm = np.random.default_rng(5).permutation(A.n).astype(np.int32)
    m = cme.Matrix(A.n, r, c, v).set_permutation(perm)
    m.pack(cme.CME_FMT_DIAG_SELL, 256, cme.CME_BAND_AUTO, cme.CME_DEVICE_HOST_ONLY)
    ref = oracle_mod.pack(oracle_mod.permute(A, perm))
    got = m.packed()
    for key in ("row_of", "slice_off", "slice_w", "val", "col", "inv_d", "lo", "up"):
        assert got[key].tobytes() == ref[key].tobytes(), key
    with pytest.raises(cme.CmeError):
        cme.Matrix(A.n, r, c, v).set_permutation(np.zeros(A.n, np.int32))


@pytest.mark.slow
def test_cfg2_toggle_full_host_parity(oracle_mod):
    """Config 2 (toggle N=224, ~100K states): enumeration, RCM, pack all bit-exact."""
    net = W.toggle_switch(224)
    a = oracle_mod.enumerate_network(net)
    b = cme.cme_network_enumerate(net)
    assert all(x.tobytes() == y.tobytes() for x, y in zip(a, b))
    states, r, c, v = a
    A = oracle_mod.ingest(len(states), r, c, v)
    assert A.n == 99908 and A.nnz == 595874
    m = host_matrix(len(states), r, c, v, cme.CME_ORDER_RCM)
    ref = oracle_mod.pack(oracle_mod.permute(A, oracle_mod.order_rcm(A)))
    got = m.packed()
    for key in ("row_of", "slice_off", "slice_w", "val", "col", "inv_d", "lo", "up"):
        assert got[key].tobytes() == ref[key].tobytes(), key
    refc = oracle_mod.compact(oracle_mod.permute(A, oracle_mod.order_rcm(A)), ref)
    refc.update(oracle_mod.value_index(ref))
    gotc = m.compact()
    assert len(gotc["dict"]) == 447 + 1   # the toggle's distinct rates + the pad value 0
    for key in refc:
        if key != "win_shift":
            assert gotc[key].tobytes() == refc[key].tobytes(), key


def test_error_paths():
    E = cme.CmeError
    with pytest.raises(E) as e:
        cme.cme_matrix_create_coo(2, [0], [1], [-1.0])
    assert e.value.status == cme.CME_ERR_NEGATIVE_RATE
    with pytest.raises(E) as e:
        cme.cme_matrix_create_coo(2, [0, 1], [1, 0], [np.nan, 1.0])
    assert e.value.status == cme.CME_ERR_INVALID_ARG
    with pytest.raises(E) as e:
        cme.cme_matrix_create_coo(3, [0, 1], [1, 0], [1.0, 1.0])
    assert e.value.status == cme.CME_ERR_ZERO_OUTFLOW
    with pytest.raises(E) as e:
        cme.cme_matrix_create_coo(2, [0, 1, 1], [1, 0, 1], [1.0, 1.0, 1.0])
    assert e.value.status == cme.CME_ERR_INVALID_ARG
    h = cme.cme_matrix_create_coo(2, [0, 1, 0, 1], [1, 0, 0, 1], [2.0, 3.0, -3.0, -2.0], cme.CME_DIAG_GIVEN)
    with pytest.raises(E) as e:      # solve before pack
        cme.cme_jacobi_solve(h, 2, None, 1e-12, 10, np.empty(2))
    assert e.value.status == cme.CME_ERR_BAD_STATE
    with pytest.raises(E) as e:      # slice must be 32
        cme._chk(cme._lib.cme_pack(h, 0, cme.cme_pack_opts(16, 256, 0, -2)), "pack")
    assert e.value.status == cme.CME_ERR_INVALID_ARG
    cme.cme_pack(h, device=cme.CME_DEVICE_HOST_ONLY)
    with pytest.raises(E) as e:      # reorder after pack
        cme.cme_reorder(h, cme.CME_ORDER_RCM)
    assert e.value.status == cme.CME_ERR_BAD_STATE
    with pytest.raises(E) as e:      # host-only layout cannot be solved
        cme.cme_jacobi_solve(h, 2, None, 1e-12, 10, np.empty(2))
    assert e.value.status == cme.CME_ERR_BAD_STATE
    with pytest.raises(E) as e:
        cme.cme_set_solver_opts(h, omega=1.5)
    assert e.value.status == cme.CME_ERR_INVALID_ARG
    with pytest.raises(E) as e:
        cme.cme_set_solver_opts(h, check_every=0)
    assert e.value.status == cme.CME_ERR_INVALID_ARG
    cme.cme_matrix_destroy(h)


def test_no_cpu_fallback_without_device():
    """On a box without a GPU the device path fails loudly (no silent CPU path)."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is visible")
    h = cme.cme_matrix_create_coo(2, [0, 1], [1, 0], [1.0, 2.0])
    with pytest.raises(cme.CmeError) as e:
        cme.cme_pack(h)
    assert e.value.status == cme.CME_ERR_NO_DEVICE
    cme.cme_matrix_destroy(h)


def test_info_bytes_model(oracle_mod):
    A = oracle_mod.network_csr(W.schnakenberg(60))
    states, r, c, v = oracle_mod.enumerate_network(W.schnakenberg(60))
    f = host_matrix(len(states), r, c, v).info()
    assert f.bytes_alg == 12 * A.nnz + 16 * A.n        # B_alg = 12 nnz + 16 n
    assert f.band_on == 1 and f.band_density > 0.99
    assert 0.9 < f.ell_efficiency <= 1.0
    assert f.bytes_fmt < f.bytes_alg                     # DIA band + separate diagonal save bytes


def _xw_case(name):
    if name == "banded-w300-irregular":
        n = 30000
        r, c, v = W.banded_markov(n, 10, 300, True, seed=5)
        return cme.Matrix(n, r, c, v), cme.CME_ORDER_NONE
    net = {"toggle90": W.toggle_switch(90), "schnakenberg40": W.schnakenberg(40)}[name]
    s, r, c, v = cme.cme_network_enumerate(net)
    return cme.Matrix(len(s), r, c, v), cme.CME_ORDER_RCM if name == "toggle90" else cme.CME_ORDER_NONE


@pytest.mark.parametrize("name", ["banded-w300-irregular", "toggle90", "schnakenberg40"])
@pytest.mark.parametrize("ncw,stages", [(16, 2), (16, 3), (30, 4)])
def test_xw_plan_invariants(name, ncw, stages):
    """The x-window plan, checked against the packed layout
    it is derived from: every row, band neighbour and gathered column of a tile
    lies in the tile's chunk range (chunk k = rows [256k - 1, 256k + 255)); both
    ends are monotone; and a replay of the producer -- tiles issued in order,
    `stages` records in flight, chunks written to slot k mod need -- never
    overwrites a chunk a live tile still reads."""
    m, order = _xw_case(name)
    m.reorder(order).pack(cme.CME_FMT_DIAG_SELL, 256, cme.CME_BAND_AUTO, cme.CME_DEVICE_HOST_ONLY)
    P = m.packed()
    plan, need, span = cme.cme_export_xw_plan(m.h, ncw, stages, P["n_slices"])
    lo, hi = plan[:, 0].astype(np.int64), plan[:, 1].astype(np.int64)
    n, T = P["n"], len(plan)
    assert np.all(np.diff(lo) >= 0) and np.all(np.diff(hi) >= 0) and np.all(hi > lo)
    chunk = lambda rows: (np.asarray(rows, np.int64) + 1) >> 8   # noqa: E731
    for t in range(T):
        q0, q1 = t * ncw, min((t + 1) * ncw, P["n_slices"])
        slots = np.arange(q0 * 32, min(q1 * 32, n))
        rows = P["row_of"][slots].astype(np.int64) if P["row_of"].size else slots
        need_rows = [rows]
        if P["band_on"]:
            need_rows += [np.maximum(rows - 1, -1), np.minimum(rows + 1, n - 1)]
        e0, e1 = P["slice_off"][q0], P["slice_off"][q1]
        need_rows.append(P["col"][e0:e1])
        k = chunk(np.concatenate(need_rows))
        assert k.min() >= lo[t] and k.max() < hi[t], (t, k.min(), k.max(), lo[t], hi[t])
    ref_need = max(hi[t] - lo[max(0, t - stages + 1)] for t in range(T))
    assert need == max(1, ref_need) and span == max(1, int((hi - lo).max()))
    # replay: ring of `need` slots, slot -> chunk currently held
    held = {}
    issued = lo[0]
    for j in range(T):
        oldest = lo[max(0, j - stages + 1)]   # tiles j-stages+1 .. j are live
        while issued < hi[j]:
            slot = issued % need
            prev = held.get(slot)
            assert prev is None or prev < oldest, (j, issued, prev, oldest)
            held[slot] = issued
            issued += 1
        for kk in range(lo[j], hi[j]):       # tile j reads chunks it finds in place
            assert held.get(kk % need) == kk
    m.close()


def test_xw_plan_errors():
    s, r, c, v = cme.cme_network_enumerate(W.toggle_switch(20))
    m = cme.Matrix(len(s), r, c, v)
    with pytest.raises(cme.CmeError) as e:          # before pack
        cme.cme_export_xw_plan(m.h, 16, 3, 1)
    assert e.value.status == cme.CME_ERR_BAD_STATE
    m.pack(device=cme.CME_DEVICE_HOST_ONLY)
    ns = m.packed()["n_slices"]
    buf = np.zeros(2 * (ns + 7), np.int32)
    need, span = cme.C.c_int64(), cme.C.c_int64()
    st = cme._lib.cme_export_xw_plan(m.h, 16, 3, ns + 7, buf.ctypes.data_as(cme.i32p), cme.C.byref(need),
                                     cme.C.byref(span))
    assert st == cme.CME_ERR_INVALID_ARG            # tiles must be ceil(n_slices / ncw)
    with pytest.raises(cme.CmeError) as e:          # ncw out of range
        cme.cme_export_xw_plan(m.h, 0, 3, ns)
    assert e.value.status == cme.CME_ERR_INVALID_ARG
    plan, need, span = cme.cme_export_xw_plan(m.h, 16, 3, ns)
    assert plan.shape == ((ns + 15) // 16, 2) and need >= span >= 1
    m.close()
