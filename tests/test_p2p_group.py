"""Row-sharded solve over the peer-memory transport, run as an
in-process group of 2-4 virtual ranks (one host thread each) on one GPU.

This exercises the whole multi-rank device path -- partition, x-span local
layouts, the step kernels' direct halo stores into the peers' buffers, the
flag barriers, the cross-rank check records and the output gather -- against
the single-GPU path and the oracle.  With several GPUs the same code stores
over NVLink.  (The NCCL transport is covered on one GPU with a 1-rank
communicator in test_gpu_parity.py and on CPU by test_partition_gloo.py.)
"""
import threading

import numpy as np
import pytest

import workloads as W

pytestmark = pytest.mark.gpu


def run_group(cme, nranks, n, r, c, v, body, order=2, window=64):
    comms = cme.cme_comm_init_local([0] * nranks)
    out, errs = [None] * nranks, []

    def worker(rank):
        try:
            m = cme.Matrix(n, r, c, v).reorder(order)
            m.pack(cme.CME_FMT_DIAG_SELL, window, cme.CME_BAND_AUTO, cme.CME_DEVICE_HOST_ONLY)
            cme.cme_matrix_distribute(m.h, comms[rank])
            out[rank] = body(m, rank)
            m.close()
        except Exception as ex:  # surfaced below
            errs.append(repr(ex))

    th = [threading.Thread(target=worker, args=(k,)) for k in range(nranks)]
    for t in th:
        t.start()
    for t in th:
        t.join(timeout=600)
    for cm in comms:
        cme.cme_comm_destroy(cm)
    assert not errs, errs
    return out


@pytest.mark.parametrize("nranks", [2, 3, 4])
@pytest.mark.parametrize("knobs", [{"CME_TMA": "0"}, {"CME_TMA": "1"}], ids=lambda k: str(k))
def test_p2p_group_solve_matches_single_gpu(oracle_mod, monkeypatch, nranks, knobs):
    import paper_conf_ipps_maggionibl13_b200 as cme
    for k, val in knobs.items():
        monkeypatch.setenv(k, val)
    states, r, c, v = oracle_mod.enumerate_network(W.toggle_switch(60))
    A = oracle_mod.ingest(len(states), r, c, v)
    n = A.n
    x = W.random_start(n, 4)

    def body(m, rank):
        info = m.info()
        m.set_opts(omega=0.9, check_every=50)
        y = m.spmv(x)
        p, st, it = m.solve(tol=1e-11, max_iter=100000)
        pt, terms = m.transient(0.2)
        return info.row_begin, info.row_end, y, p, st, it, pt

    res = run_group(cme, nranks, n, r, c, v, body)
    cuts = sorted((a, b) for a, b, *_ in res)
    assert cuts[0][0] == 0 and cuts[-1][1] == n and all(cuts[i][1] == cuts[i + 1][0] for i in range(nranks - 1))
    yref = oracle_mod.jacobi_step(A, x, 0.9)
    single = cme.Matrix(n, r, c, v).reorder(2).pack(cme.CME_FMT_DIAG_SELL, 64)
    single.set_opts(omega=0.9, check_every=50)
    p1, st1, it1 = single.solve(tol=1e-11, max_iter=100000)
    o = oracle_mod.jacobi_solve(A, omega=0.9, tol=0.0, check_every=50, max_iter=it1)
    ptr, _, _ = oracle_mod.transient(A, 0.2)
    for _, _, y, p, st, it, pt in res:
        assert np.max(np.abs(y - yref) / yref) <= 1e-13
        assert st == st1 == "CONVERGED" and it == it1
        assert np.abs(p - p1).sum() <= 1e-13 and np.abs(p - o.p).sum() <= 1e-10
        assert np.abs(pt - ptr).sum() <= 1e-12


def test_p2p_group_batch_and_fixed_iterations(oracle_mod):
    import paper_conf_ipps_maggionibl13_b200 as cme
    nets = [W.toggle_switch(40, s=50.0 * f) for f in (1.0, 1.4)]
    coos = [oracle_mod.enumerate_network(net) for net in nets]
    states, r, c, _ = coos[0]
    n = len(states)
    rates = np.stack([co[3] for co in coos])
    As = [oracle_mod.ingest(n, r, c, co[3]) for co in coos]

    def body(m, rank):
        m.set_opts(omega=0.9, check_every=25, stag_tol=0.0)
        p, st, it = m.solve(tol=0.0, max_iter=210)
        return p, st, it

    for p, st, it in run_group(cme, 2, n, r, c, rates, body):
        assert st == "NOT_CONVERGED" and it == 210
        for b in range(2):
            o = oracle_mod.jacobi_solve(As[b], omega=0.9, tol=0.0, check_every=25, max_iter=210, stag_tol=0.0)
            assert np.abs(p[b * n:(b + 1) * n] - o.p).sum() <= 1e-12


@pytest.mark.parametrize("nranks", [2, 4, 8])
@pytest.mark.parametrize("fused", ["1", "0"])
def test_fused_halo_sync_virtual_ranks(oracle_mod, monkeypatch, nranks, fused):
    """The fused in-kernel halo sync: the tile-record step
    kernel gates its boundary tiles on the peers' pushed / consumed step
    counts instead of a flag-barrier kernel after every step.  2, 4 and 8
    virtual ranks share one GPU, each rank's grid capped to its share of the
    SMs so all ranks' step kernels are resident together (a gate spins until
    a peer's tiles have run).  SpMV, a fixed-iteration run, a converged solve
    and a transient vs the single-GPU path and the oracle; CME_P2P_FUSED = 0
    (per-step neighbour barrier) on the same cases."""
    import paper_conf_ipps_maggionibl13_b200 as cme
    for k, val in {"CME_TMA": "1", "CME_RESIDENT": "0", "CME_P2P_FUSED": fused}.items():
        monkeypatch.setenv(k, val)
    states, r, c, v = oracle_mod.enumerate_network(W.toggle_switch(150))
    A = oracle_mod.ingest(len(states), r, c, v)
    n = A.n
    x = W.random_start(n, 6)

    def body(m, rank):
        info = m.info()
        m.set_opts(omega=0.9, check_every=40, stag_tol=0.0)
        y = m.spmv(x)
        pf, stf, itf = m.solve(tol=0.0, max_iter=130)
        m.set_opts(omega=0.9, check_every=100)
        p, st, it = m.solve(tol=1e-10, max_iter=100000)
        pt, terms = m.transient(0.1)
        return info.halo_fused, info.records, y, pf, itf, p, st, it, pt

    res = run_group(cme, nranks, n, r, c, v, body, window=256)
    yref = oracle_mod.jacobi_step(A, x, 0.9)
    of = oracle_mod.jacobi_solve(A, omega=0.9, tol=0.0, check_every=40, max_iter=130, stag_tol=0.0)
    single = cme.Matrix(n, r, c, v).reorder(2).pack(cme.CME_FMT_DIAG_SELL, 256)
    single.set_opts(omega=0.9, check_every=100)
    p1, st1, it1 = single.solve(tol=1e-10, max_iter=100000)
    ptr, _, _ = oracle_mod.transient(A, 0.1)
    for hf, rec, y, pf, itf, p, st, it, pt in res:
        assert rec == 1 and hf == int(fused)
        assert np.max(np.abs(y - yref) / yref) <= 1e-13
        assert itf == 130 and np.abs(pf - of.p).sum() <= 1e-12
        assert st == st1 == "CONVERGED" and it == it1
        assert np.abs(p - p1).sum() <= 1e-13
        assert np.abs(pt - ptr).sum() <= 1e-12
