"""Batched parameter sweeps (the same network
under different conditions).  B rate sets share one pattern; every member
must equal the oracle run on that member alone -- the batch is B independent
instances of the plain definition, so no new oracle code is involved.

CPU: the packed batch layout is bit-exact against the oracle's per-member
packs (values member-minor, pattern arrays shared).  GPU: per-member SpMV
parity (<= 1e-13) and landscape parity (<= 1e-10 L1) on every step kernel.
"""
import numpy as np
import pytest

import paper_conf_ipps_maggionibl13_b200 as cme
import workloads as W


def toggle_members(N, B):
    """B toggle switches that differ in synthesis/degradation/binding rates."""
    fac = [1.0, 0.7, 1.3, 2.0, 0.5, 1.1, 0.9, 1.6][:B]
    return [W.toggle_switch(N, s=50.0 * f, d=1.0 / f ** 0.5, b=0.005 * f, u=0.1) for f in fac]


def batch_inputs(oracle_mod, nets):
    coos = [oracle_mod.enumerate_network(n) for n in nets]
    states, r, c, _ = coos[0]
    for s2, r2, c2, _ in coos[1:]:
        assert np.array_equal(states, s2) and np.array_equal(r, r2) and np.array_equal(c, c2)
    rates = np.stack([v for *_, v in coos])
    As = [oracle_mod.ingest(len(states), r, c, v) for *_, v in coos]
    return len(states), r, c, rates, As


@pytest.mark.parametrize("B", [2, 4, 8])
@pytest.mark.parametrize("order,window,band", [("rcm", 256, "auto"), ("none", 1, "always"), ("dfs", 64, "never")])
def test_batch_pack_bit_exact(oracle_mod, B, order, window, band):
    n, r, c, rates, As = batch_inputs(oracle_mod, toggle_members(17, B))
    om = {"none": 0, "dfs": 1, "rcm": 2}[order]
    bm = {"auto": 0, "always": 1, "never": 2}[band]
    m = cme.Matrix(n, r, c, rates).reorder(om)
    m.pack(cme.CME_FMT_DIAG_SELL, window, bm, cme.CME_DEVICE_HOST_ONLY)
    got = m.packed()
    assert got["batch"] == B and m.info().batch == B
    perm = {"none": np.arange(n, dtype=np.int32), "dfs": oracle_mod.order_dfs(As[0], 0),
            "rcm": oracle_mod.order_rcm(As[0])}[order]
    assert np.array_equal(m.permutation(), perm)
    for b in range(B):
        ref = oracle_mod.pack(oracle_mod.permute(As[b], perm), window=window, band=band)
        for key in ("row_of", "slice_off", "slice_w", "col"):
            assert got[key].tobytes() == ref[key].tobytes(), key
        for key in ("val", "inv_d", "lo", "up"):
            assert got[key][b::B].tobytes() == ref[key].tobytes(), (key, b)
    # shared offsets + value index of the members' B-tuples,
    # bit-exact against the oracle's definition applied to the oracle packs
    refs = [oracle_mod.pack(oracle_mod.permute(As[b], perm), window=window, band=band) for b in range(B)]
    Pb = dict(refs[0])
    Pb["batch"] = B
    for key in ("val", "lo", "up"):
        Pb[key] = np.stack([rf[key] for rf in refs], axis=1).reshape(-1)
    gotc = m.compact()
    refc = oracle_mod.compact(oracle_mod.permute(As[0], perm), refs[0])   # offsets: member-independent
    for key in ("col16", "row8"):
        if key in refc:
            assert gotc[key].tobytes() == refc[key].tobytes(), key
    refv = oracle_mod.value_index(Pb)
    assert refv is not None and "val" not in gotc
    for key, v in refv.items():
        assert gotc[key].dtype == v.dtype and gotc[key].tobytes() == v.tobytes(), key
    # each entry's tuple reproduces every member's stored value
    d = gotc["dict"].reshape(-1, B)
    assert d[gotc["vidx"]].reshape(-1).tobytes() == got["val"].tobytes()


def test_batch_union_pattern_with_member_zeros(oracle_mod):
    """An entry zero in one member but not another is stored (the pattern is
    the union); each member's matrix is still its own A (dense comparison)."""
    rng = np.random.default_rng(3)
    n = 60
    r = np.concatenate([(np.arange(n) + 1) % n, rng.integers(0, n, 300)]).astype(np.int32)
    c = np.concatenate([np.arange(n), rng.integers(0, n, 300)]).astype(np.int32)
    keep = r != c
    r, c = r[keep], c[keep]
    rates = rng.random((2, len(r))) + 0.1
    rates[1, n:][rng.random(len(r) - n) < 0.5] = 0.0       # member 1 drops half the extra entries
    m = cme.Matrix(n, r, c, rates).pack(device=cme.CME_DEVICE_HOST_ONLY)
    P = m.packed()
    for b in range(2):
        A = oracle_mod.ingest(n, r, c, rates[b])
        D = np.zeros((n, n))
        for s in range(n):
            q, lane = divmod(s, 32)
            row = P["row_of"][s]
            D[row, row] = -1.0 / P["inv_d"][s * 2 + b]
            if P["band_on"]:
                if row > 0:
                    D[row, row - 1] += P["lo"][s * 2 + b]
                if row + 1 < n:
                    D[row, row + 1] += P["up"][s * 2 + b]
            for t in range(P["slice_w"][q]):
                e = P["slice_off"][q] + lane + 32 * t
                if P["col"][e] != row or P["val"][e * 2 + b] != 0.0:
                    D[row, P["col"][e]] += P["val"][e * 2 + b]
        ref = A.dense()
        assert np.allclose(D, ref, rtol=1e-15, atol=0)


def test_batch_errors():
    with pytest.raises(cme.CmeError):
        cme.Matrix(3, [0, 1, 2], [1, 2, 0], np.ones((3, 3)))         # batch 3 unsupported
    with pytest.raises(cme.CmeError) as e:
        cme.Matrix(3, [0, 1, 2], [1, 2, 0], np.array([[1.0, 1, 1], [1, 0, 1]]))   # member 1: state 1 no outflow
    assert e.value.status == cme.CME_ERR_ZERO_OUTFLOW
    m = cme.Matrix(3, [0, 1, 2], [1, 2, 0], np.ones((2, 3)))
    with pytest.raises(cme.CmeError):
        m.pack(cme.CME_FMT_CSR, device=cme.CME_DEVICE_HOST_ONLY)


# ------------------------------------------------------------------ GPU -------

KNOBS = [{"CME_TMA": "0"}, {"CME_TMA": "1", "CME_VI": "0"}, {"CME_TMA": "1", "CME_TMA_WARPS": "8", "CME_VI": "0"},
         {"CME_TMA": "1", "CME_VI2B": "0"}, {"CME_TMA": "1", "CME_TMA_WARPS": "8", "CME_VI2B": "0"},
         {"CME_TMA": "1", "CME_TMA_WARPS": "15", "CME_VI2B": "0"},   # batched value index (sell_vib_kernel)
         {"CME_TMA": "1"},                                            # auto: the records at B = 2
         {"CME_TMA": "1", "CME_VI2B": "1"},                           # its tile records (sell_vi2b_kernel)
         {"CME_TMA": "1", "CME_VI2B": "1", "CME_VI2B_SD": "0"},       # (B = 2: tuples through L1, not staged)
         {"CME_TMA": "1", "CME_VI2B": "1", "CME_VI2_WARPS": "alt"},
         {"CME_TMA": "1", "CME_VI2B": "1", "CME_VI2_GRID": "3", "CME_VI2_STAGES": "2"}]   # ring wraps many times
ALT_WARPS = {2: "30", 4: "30", 8: "8"}   # sell_vi2b_kernel's second shape per B


@pytest.mark.gpu
@pytest.mark.parametrize("B", [2, 4, 8])
@pytest.mark.parametrize("knobs", KNOBS, ids=lambda k: ",".join(f"{a}={b}" for a, b in k.items()))
def test_batch_spmv_and_landscape_parity(oracle_mod, monkeypatch, B, knobs):
    for k, v in knobs.items():
        monkeypatch.setenv(k, ALT_WARPS[B] if v == "alt" else v)
    n, r, c, rates, As = batch_inputs(oracle_mod, toggle_members(26, B))
    m = cme.Matrix(n, r, c, rates).reorder(cme.CME_ORDER_RCM).pack()
    f = m.info()
    assert f.kernel == (1 if knobs["CME_TMA"] == "1" else 0)
    assert f.compact == (2 if knobs["CME_TMA"] == "1" and knobs.get("CME_VI") != "0" else 0)
    if "CME_TMA_WARPS" in knobs:
        assert f.tma_warps == int(knobs["CME_TMA_WARPS"])
    records = knobs["CME_TMA"] == "1" and knobs.get("CME_VI") != "0" and (
        knobs.get("CME_VI2B") == "1" or (knobs.get("CME_VI2B") is None and B == 2))
    assert f.records == int(records), (f.records, knobs)
    if knobs.get("CME_VI2_WARPS") == "alt":
        assert f.tma_warps == int(ALT_WARPS[B])
    if "CME_VI2_GRID" in knobs:
        assert f.grid <= 3
    m.set_opts(omega=0.9, check_every=7, stag_tol=0.0)
    x = np.concatenate([W.random_start(n, 30 + b) for b in range(B)])
    y = m.spmv(x)
    for b in range(B):
        ref = As[b]
        yr = oracle_mod.jacobi_step(ref, x[b * n:(b + 1) * n], 0.9)
        yb = y[b * n:(b + 1) * n]
        assert np.max(np.abs(yb - yr) / yr) <= 1e-13
    p, st, it = m.solve(tol=1e-11, max_iter=200000)
    assert st == "CONVERGED"
    reps = m.batch_report()
    for b in range(B):
        o = oracle_mod.jacobi_solve(As[b], omega=0.9, tol=1e-11, check_every=7, stag_tol=0.0)
        assert o.status == "CONVERGED" and reps[b].status == cme.CME_OK
        assert abs(reps[b].iters - o.iters) <= 7
        o2 = oracle_mod.jacobi_solve(As[b], omega=0.9, tol=0.0, check_every=7, max_iter=it, stag_tol=0.0)
        assert np.abs(p[b * n:(b + 1) * n] - o2.p).sum() <= 1e-10
    assert it == max(rp.iters for rp in reps)


@pytest.mark.gpu
def test_batch_p0_and_device_vectors(oracle_mod):
    import torch
    n, r, c, rates, As = batch_inputs(oracle_mod, toggle_members(20, 4))
    m = cme.Matrix(n, r, c, rates).reorder(cme.CME_ORDER_RCM).pack()
    m.set_opts(omega=0.9, check_every=50, stag_tol=0.0)
    p0 = torch.tensor(np.concatenate([W.random_start(n, b) for b in range(4)]), device="cuda")
    out = torch.empty(4 * n, dtype=torch.float64, device="cuda")
    m.solve(p0=p0, tol=0.0, max_iter=333, p_out=out)
    out = out.cpu().numpy()
    for b in range(4):
        o = oracle_mod.jacobi_solve(As[b], p0=p0[b * n:(b + 1) * n].cpu().numpy(), omega=0.9, tol=0.0,
                                    check_every=50, max_iter=333, stag_tol=0.0)
        assert np.abs(out[b * n:(b + 1) * n] - o.p).sum() <= 1e-12


@pytest.mark.gpu
@pytest.mark.parametrize("B", [2, 4, 8])
def test_batch_records_bit_identical_to_sell_vib(oracle_mod, monkeypatch, B):
    """The batched tile records (sell_vi2b_kernel) do sell_vib_kernel's
    arithmetic exactly (same tuples, FMA order, row sum times inv_d): their
    SpMVs agree bit for bit."""
    n, r, c, rates, _ = batch_inputs(oracle_mod, toggle_members(30, B))
    x = np.concatenate([W.random_start(n, 40 + b) for b in range(B)])
    out = {}
    for rec in ("0", "1"):
        monkeypatch.setenv("CME_TMA", "1")
        monkeypatch.setenv("CME_VI2B", rec)   # (1 forces the records at every B)
        m = cme.Matrix(n, r, c, rates).reorder(cme.CME_ORDER_RCM).pack()
        assert m.info().records == int(rec)
        m.set_opts(omega=0.9)
        out[rec] = m.spmv(x)
        m.close()
    assert np.array_equal(out["0"], out["1"])
