"""Peer-memory transport across PROCESSES: cme_comm_init_ipc,
buffers exported as CUDA IPC handles, blobs all-gathered over a gloo group,
cme_matrix_ipc_attach -- the path bench.py takes under torchrun.

Both processes share the one GPU of the test box (the driver time-slices the
two contexts, so every flag barrier waits for the other process's slice: slow
per iteration, but the data path is the multi-GPU one).  Results must equal the
single-process solve and the oracle.
"""
import multiprocessing as mp
import socket

import numpy as np
import pytest

import workloads as W

pytestmark = pytest.mark.gpu

ITERS = 120


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, n, r, c, v, x, q):
    try:
        import torch
        import torch.distributed as dist
        import paper_conf_ipps_maggionibl13_b200 as cme
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
        comm = cme.cme_comm_init_ipc(world, rank, 0)
        m = cme.Matrix(n, r, c, v).reorder(cme.CME_ORDER_RCM)
        m.pack(cme.CME_FMT_DIAG_SELL, 64, cme.CME_BAND_AUTO, cme.CME_DEVICE_HOST_ONLY)
        cme.cme_matrix_distribute(m.h, comm)
        blobs = [None] * world
        dist.all_gather_object(blobs, cme.cme_matrix_ipc_export(m.h))
        cme.cme_matrix_ipc_attach(m.h, blobs)
        m.set_opts(omega=0.9, check_every=30, stag_tol=0.0)
        y = m.spmv(x)
        p, st, it = m.solve(tol=0.0, max_iter=ITERS)
        info = m.info()
        dist.barrier()   # peers stop touching my buffers before I free them
        m.close()
        cme.cme_comm_destroy(comm)
        dist.destroy_process_group()
        q.put((rank, info.row_begin, info.row_end, y, p, st, it, None))
    except Exception as ex:  # surfaced in the parent
        q.put((rank, 0, 0, None, None, None, None, repr(ex)))


def test_ipc_two_processes_match_oracle(oracle_mod):
    states, r, c, v = oracle_mod.enumerate_network(W.toggle_switch(50))
    A = oracle_mod.ingest(len(states), r, c, v)
    n = A.n
    x = W.random_start(n, 9)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(k, 2, port, n, r, c, v, x, q)) for k in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=900) for _ in procs]
    for p in procs:
        p.join(timeout=120)
    errs = [e for *_, e in res if e]
    assert not errs, errs
    res.sort(key=lambda t: t[0])
    assert res[0][1] == 0 and res[0][2] == res[1][1] and res[1][2] == n
    yref = oracle_mod.jacobi_step(A, x, 0.9)
    o = oracle_mod.jacobi_solve(A, omega=0.9, tol=0.0, check_every=30, max_iter=ITERS, stag_tol=0.0)
    for _, _, _, y, p, st, it, _ in res:
        assert np.max(np.abs(y - yref) / yref) <= 1e-13
        assert st == "NOT_CONVERGED" and it == ITERS
        assert np.abs(p - o.p).sum() <= 1e-12


def test_ipc_attach_required_before_solve(oracle_mod):
    import paper_conf_ipps_maggionibl13_b200 as cme
    states, r, c, v = oracle_mod.enumerate_network(W.toggle_switch(10))
    comm = cme.cme_comm_init_ipc(1, 0, 0)
    m = cme.Matrix(len(states), r, c, v)
    m.pack(cme.CME_FMT_DIAG_SELL, 64, cme.CME_BAND_AUTO, cme.CME_DEVICE_HOST_ONLY)
    cme.cme_matrix_distribute(m.h, comm)
    with pytest.raises(cme.CmeError, match="BAD_STATE|bad state|attach"):
        m.solve(tol=1e-9, max_iter=100)
    cme.cme_matrix_ipc_attach(m.h, [cme.cme_matrix_ipc_export(m.h)])
    p, st, _ = m.solve(tol=1e-9, max_iter=100000)
    assert st == "CONVERGED" and abs(p.sum() - 1) < 1e-12
    m.close()
    cme.cme_comm_destroy(comm)
