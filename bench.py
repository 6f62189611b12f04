#!/usr/bin/env python3
"""Benchmark of the CME steady-state Jacobi hot path (BASELINE.json metric:
fp64 Jacobi GFLOPS & iters/s, % HBM roofline, time-to-converge at 1/2/4/8 B200).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config NAME] [--impl reference]

One STEP = one check block of C = 100 fused Jacobi iterations (SURVEY 8(a)
rows a4 + a5, plus a6 halo/scalar collectives when N > 1) over the resident
matrix of the workload; ingest/reorder/pack (a1-a3) are one-time setup
("neglected ... amortizing this one-time cost") and a7 (un-permute +
D2H) is inside the e2e leg.  GFLOPS counts 2 nnz(A) flops per iteration, the
paper's convention (reading R15).

Default workload: configs[3] "toggle switch with enlarged
molecule buffer, ~20M states" (N = 3164: n = 20,015,468, nnz = 120,042,194),
RCM order, DIAG+SELL layout, omega = 0.9 -- the >= 10M-state network of the
north-star target, whose 1.76 GB/iteration exceeds the 126 MB L2 (no flush
needed).  configs[1] (~100K states, L2-resident) is reported as the
time-to-converge line in "converge"; configs[2] (Schnakenberg, 2M states) is solved to
tol 1e-12 and compared with its closed form in "converge_closed_form".

--impl reference times the oracle (oracle/, plain C, all host cores) on the
same workload and metric: the reference arm of this paper-only tier.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import tempfile
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

# one process per GPU: split the host cores between the ranks for the host
# setup (enumeration, ingest, RCM, pack use OpenMP) before any library loads
if int(os.environ.get("WORLD_SIZE", "1")) > 1 and "OMP_NUM_THREADS" not in os.environ:
    _lw = max(1, int(os.environ.get("LOCAL_WORLD_SIZE", os.environ["WORLD_SIZE"])))
    os.environ["OMP_NUM_THREADS"] = str(max(1, len(os.sched_getaffinity(0)) // _lw))

import workloads as W  # noqa: E402

C_BLOCK = 100
DEFAULTS = {
    "cfg4_toggle_20m": dict(order="rcm", window=256, omega=0.9),
    "cfg3a_schnakenberg_2m": dict(order="none", window=256, omega=1.0),
    "cfg3b_brusselator_2m": dict(order="none", window=256, omega=0.9),
    "cfg2_toggle_100k": dict(order="rcm", window=256, omega=0.9),
}


_T0 = time.time()


def log(*a):
    print(f"[{time.time() - _T0:7.1f}s]", *a, file=sys.stderr, flush=True)


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f)
    except OSError:
        return {}


def hbm_peak():
    pk = measured_peaks()
    if "hbm_gbs" in pk:
        return float(pk["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def ncu_traffic(workload, kernel):
    """dram bytes/launch of the step kernel from the committed ncu --set full
    capture (profiles/ncu_summary.json), only if it was taken of this kernel;
    returns (bytes, "committed ncu capture @ <commit>: <kernel>")."""
    p = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        with open(p) as f:
            d = json.load(f).get(workload, {})
    except (OSError, ValueError):
        return None, None
    if not d.get("dram_bytes_per_launch") or d.get("kernel_short") != kernel:
        return None, "no committed ncu capture of this kernel"
    return d["dram_bytes_per_launch"], f"committed ncu capture @ {d.get('commit', '?')}: {d.get('kernel')}"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled DURING the timed region."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index):
        self.idx = gpu_index
        self.proc = None
        self.f = None

    def __enter__(self):
        try:
            self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.idx}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=self.f, stderr=subprocess.DEVNULL)
            time.sleep(0.3)
        except (OSError, FileNotFoundError):
            self.proc = None
        return self

    def __exit__(self, *exc):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self):
        if not self.f:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.f.flush()
        rows = []
        with open(self.f.name) as g:
            for line in g:
                parts = [x.strip() for x in line.split(",")]
                if len(parts) >= 9 and parts[1].isdigit():
                    rows.append(parts)
        os.unlink(self.f.name)
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        sm = sorted(int(r[1]) for r in rows)
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[5 + i].lower().startswith("active")})
        return {"sm_mhz": sm[len(sm) // 2], "sm_max_mhz": int(rows[0][2]), "reasons": reasons,
                "samples": len(rows), "power_w_max": max(float(r[3]) for r in rows if r[3] not in ("", "[N/A]"))}


def kernel_name(info):
    if info.kernel == 1 and getattr(info, "records", 0):
        return f"sell_vi2_kernel<{info.tma_warps}>"
    if info.kernel == 1 and info.compact == 2:
        return f"sell_vi_kernel<{info.tma_warps}>"
    if info.kernel == 1 and info.compact:
        return f"sell_cpt_kernel<{info.tma_warps}>"
    return {0: "sell_step_kernel", 1: f"sell_tma_kernel<{info.tma_warps}>", 2: "csr_step_kernel",
            3: "sell_resident_kernel"}.get(
        info.kernel, "?")


def build_matrix(cme, name, dev_mode, batch=1, first=0):
    cfg = DEFAULTS[name]
    t0 = time.perf_counter()
    if batch > 1 or first > 0:   # sweep members first .. first+B-1: B rate sets on one pattern
        vs = []
        for net in W.sweep_networks(name, batch, first):
            states, r, c, v = cme.cme_network_enumerate(net)
            vs.append(v)
        v = np.stack(vs) if batch > 1 else vs[0]
    else:
        states, r, c, v = cme.cme_network_enumerate(W.config_network(name))
    t1 = time.perf_counter()
    n = len(states)
    m = cme.Matrix(n, r, c, v)
    m.states = states
    del r, c, v
    m.reorder({"none": cme.CME_ORDER_NONE, "dfs": cme.CME_ORDER_DFS, "rcm": cme.CME_ORDER_RCM}[cfg["order"]])
    t2 = time.perf_counter()
    m.pack(cme.CME_FMT_DIAG_SELL, cfg["window"], cme.CME_BAND_AUTO, dev_mode)
    t3 = time.perf_counter()
    setup = {"enumerate_s": round(t1 - t0, 2), "ingest_reorder_s": round(t2 - t1, 2), "pack_upload_s": round(t3 - t2, 2)}
    return m, cfg, setup


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def oracle_run(oracle, A, iters, omega, nthreads):
    """One oracle call of `iters` Jacobi iterations (one check block of `iters`)."""
    t = time.perf_counter()
    oracle.jacobi_solve(A, omega=omega, tol=0.0, check_every=iters, max_iter=iters, stag_tol=0.0, nthreads=nthreads)
    return time.perf_counter() - t


def cpu_oracle_timing(name, budget_s=20.0, omega=0.9, budget_1t_s=10.0):
    """Time the oracle (plain C CSR Jacobi, as it stands) on a bounded sample of
    the workload -- one call of up to C = 100 iterations of the full matrix on
    all host cores, and a shorter one on 1 thread (both thread
    counts and the CPU model).  The calls include the oracle's own per-call
    setup (norm, iterate allocation), amortised over the sample."""
    import oracle
    net = W.config_network(name)
    t0 = time.perf_counter()
    A = oracle.network_csr(net)
    t_setup = time.perf_counter() - t0
    cores = len(os.sched_getaffinity(0))
    one = max(oracle_run(oracle, A, 2, omega, cores) / 2, 1e-6)            # calibrate
    iters = int(max(2, min(C_BLOCK, budget_s / one)))
    tt = oracle_run(oracle, A, iters, omega, cores)
    one1 = max(oracle_run(oracle, A, 1, omega, 1), 1e-6)
    iters1 = int(max(1, min(C_BLOCK, budget_1t_s / one1)))
    tt1 = oracle_run(oracle, A, iters1, omega, 1)
    gflops = 2.0 * A.nnz * iters / tt / 1e9
    return dict(value=round(gflops, 4), unit="GFLOPS", cores=cores, kind="oracle",
                sample=f"{iters} Jacobi iterations of the full {name} matrix (n={A.n}, nnz={A.nnz}) in one oracle "
                       f"call (plain C CSR, OpenMP {cores} threads); 1-thread: {iters1} iterations",
                cpu_model=cpu_model(), iters_per_s=round(iters / tt, 3), seconds_per_iter=tt / iters,
                value_1thread=round(2.0 * A.nnz * iters1 / tt1 / 1e9, 4), iters_per_s_1thread=round(iters1 / tt1, 3),
                oracle_setup_s=round(t_setup, 1))


def run_reference(args):
    """The reference arm of this paper-only tier: the oracle (plain C, CPU, all
    host cores) timed as it stands on the same workload and metric.  A step is
    one check block of C = 100 iterations (fewer only if 100 would not fit the
    few-minute budget -- then iters_per_step says how many); warm-up and timed
    steps each run as ONE oracle call of W (K) blocks with its check every
    block, so ms_per_step is measured, not extrapolated, and the call's setup
    (||A||_inf, allocations) is amortised over the K steps."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle
    name = args.config
    omega = DEFAULTS[name]["omega"]
    A = oracle.network_csr(W.config_network(name))   # setup: not timed
    cores = len(os.sched_getaffinity(0))
    one = max(oracle_run(oracle, A, 2, omega, cores) / 2, 1e-6)
    budget = float(os.environ.get("CME_REF_BUDGET_S", "240"))
    per_step = int(max(1, min(C_BLOCK, budget / one / (args.steps + args.warmup))))

    def blocks(k):
        t = time.perf_counter()
        oracle.jacobi_solve(A, omega=omega, tol=0.0, check_every=per_step, max_iter=k * per_step, stag_tol=0.0,
                            nthreads=cores)
        return time.perf_counter() - t

    blocks(args.warmup)
    sec = blocks(args.steps)
    iters = args.steps * per_step
    gflops = 2.0 * A.nnz * iters / sec / 1e9
    line = {"metric": "fp64 Jacobi GFLOPS (2 nnz/iteration)", "value": round(gflops, 4), "unit": "GFLOPS",
            "impl": "reference", "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(sec / args.steps * 1e3, 3), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": name, "iters_per_step": per_step, "check_every": per_step,
                       "reference": "oracle/ (plain C CSR Jacobi, CPU)"},
            "cpu_baseline": {"value": round(gflops, 4), "unit": "GFLOPS", "cores": cores, "kind": "oracle",
                             "sample": f"{args.steps} steps x {per_step} Jacobi iterations of the full {name} matrix "
                                       f"(n={A.n}, nnz={A.nnz}) in one oracle call, OpenMP {cores} threads",
                             "cpu_model": cpu_model()},
            "e2e": {"value": round(gflops, 4), "unit": "GFLOPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
            "iters_per_s": round(iters / sec, 3)}
    print(json.dumps(line), flush=True)
    return 0


def converge_line(cme, name="cfg2_toggle_100k", tol=1e-12):
    """configs[1]: time-to-converge of the ~100K-state toggle on 1 GPU (resident matrix)."""
    m, cfg, setup = build_matrix(cme, name, -1)
    m.set_opts(omega=cfg["omega"], check_every=C_BLOCK)
    m.solve(tol=tol, max_iter=200000)   # warm (graph build / first resident launch)
    t = time.perf_counter()
    p, st, it = m.solve(tol=tol, max_iter=200000)
    wall = time.perf_counter() - t
    rep = m.report()
    info = m.info()
    out = {"workload": name, "n": info.n, "nnz": info.nnz, "tol": tol, "omega": cfg["omega"], "status": st,
           "iters": it, "device_seconds": round(rep.seconds, 6), "wall_seconds": round(wall, 6),
           "iters_per_s": round(it / rep.seconds, 1) if rep.seconds > 0 else None,
           "gflops": round(2 * info.nnz * it / rep.seconds / 1e9, 2) if rep.seconds > 0 else None}
    m.close()
    return out


def solve_paper_mode(cme, m, name, omega, eps=1e-8):
    """The paper's own stop test (reading R21):
    ||A p||_inf / (||A||_inf ||p||_inf) <= eps = 1e-8, checked every C = 100
    iterations, from uniform p0 -- the Table IV convention."""
    m.set_opts(omega=omega, check_every=C_BLOCK, stop=cme.CME_STOP_PAPER_RESID)
    t = time.perf_counter()
    p, st, it = m.solve(tol=eps, max_iter=200_000)
    wall = time.perf_counter() - t
    rep = m.report()
    log(f"[bench] paper mode {name}: {st} after {it} iterations, {wall:.1f}s")
    m.set_opts(omega=omega, check_every=C_BLOCK, stop=cme.CME_STOP_DELTA_L1)
    return {"workload": name, "stop": "paper residual ||Ap||_inf/(||A||_inf ||p||_inf) (P:L117)", "eps": eps,
            "check_every": C_BLOCK, "omega": omega, "status": st, "iters": it, "resid": rep.resid,
            "delta": rep.delta, "device_seconds": round(rep.seconds, 4), "wall_seconds": round(wall, 4)}


def converge_closed_form(cme, name="cfg3a_schnakenberg_2m", tol=1e-12):
    """configs[2] (Schnakenberg, n = 2,003,001, Table I size) solved to tol on 1 GPU,
    plus its L1 distance to the exact stationary law: the network satisfies
    detailed balance, so pi(x, y) is product Poisson with means k1/k2 and
    k3/k4, evaluated in log space."""
    import math
    from scipy.special import gammaln
    m, cfg, setup = build_matrix(cme, name, -1)
    m.set_opts(omega=cfg["omega"], check_every=C_BLOCK)
    t = time.perf_counter()
    p, st, it = m.solve(tol=tol, max_iter=2_000_000)
    wall = time.perf_counter() - t
    log(f"[bench] {name}: {st} after {it} iterations, {wall:.1f}s")
    rep = m.report()
    info = m.info()
    meta = W.config_network(name).meta
    S = m.states.astype(np.float64)
    a, b = meta["k1"] / meta["k2"], meta["k3"] / meta["k4"]
    logs = S[:, 0] * math.log(a) - gammaln(S[:, 0] + 1) + S[:, 1] * math.log(b) - gammaln(S[:, 1] + 1)
    pi = np.exp(logs - logs.max())
    pi /= pi.sum()
    out = {"workload": name, "n": info.n, "nnz": info.nnz, "tol": tol, "omega": cfg["omega"], "status": st,
           "iters": it, "device_seconds": round(rep.seconds, 4), "wall_seconds": round(wall, 4),
           "iters_per_s": round(it / rep.seconds, 1) if rep.seconds > 0 else None,
           "gflops": round(2 * info.nnz * it / rep.seconds / 1e9, 2) if rep.seconds > 0 else None,
           "kernel": kernel_name(info), "l1_to_closed_form": float(np.abs(p - pi).sum()),
           "closed_form": "product Poisson (detailed balance), means k1/k2, k3/k4",
           "paper_mode": solve_paper_mode(cme, m, name, cfg["omega"])}
    m.close()
    return out


def replica_members(rank, batch):
    """Replicas (`--replicas`): rank r solves sweep members [r B, r B + B) on its
    own GPU -- independent problems, no data-path collective (P:L5, L17, L83:
    the same network under different conditions)."""
    return list(range(rank * batch, rank * batch + batch))


def aggregate(dist, world, dev, ms, work):
    """Whole-job numbers of a multi-rank run: the slowest rank's time and the
    work of all ranks (flops), so value = total work / max time."""
    if world == 1:
        return ms, work
    import torch
    t = torch.tensor([ms], device=dev, dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    w = torch.tensor([work], device=dev, dtype=torch.float64)
    dist.all_reduce(w, op=dist.ReduceOp.SUM)
    return float(t.item()), float(w.item())


def self_launch(nproc):
    """`bench.py --gpus N` outside torchrun: launch the N ranks ourselves (one
    process per GPU, the launcher the driver uses, rendezvous on 127.0.0.1)
    instead of silently measuring one GPU.  Rank 0 prints the JSON line."""
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={nproc}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
    log("[bench] --gpus", nproc, "without torchrun: launching", " ".join(cmd[2:6]))
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=30)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="cfg4_toggle_20m", choices=sorted(DEFAULTS))
    ap.add_argument("--impl", default="cme", choices=["cme", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-converge", action="store_true")
    ap.add_argument("--batch", type=int, default=1, choices=[1, 2, 4, 8],
                    help="solve a sweep of B rate sets on the workload's pattern (SURVEY NEXT-1)")
    ap.add_argument("--replicas", action="store_true",
                    help="with --gpus N: every rank solves its own members of a parameter sweep on its own GPU "
                         "(weak scaling, no data-path collective) instead of row-sharding one matrix")
    ap.add_argument("--transport", choices=["p2p", "nccl"], default=os.environ.get("CME_TRANSPORT", "p2p"),
                    help="multi-rank halo/record exchange: peer-memory stores from the step kernel + flag "
                         "barriers over CUDA IPC (p2p), or NCCL send/recv + allgather in the graphs (nccl)")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.gpus > 1 and "RANK" not in os.environ:
        return self_launch(args.gpus)
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist
    world = int(os.environ.get("WORLD_SIZE", "1"))
    # under torchrun (RANK set) the row-sharded path runs even with one rank:
    # communicator, distribute, halo/record exchange in the graphs
    dist_path = "RANK" in os.environ
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # more ranks than GPUs (a one-GPU test box only): ranks share the GPUs over
    # the peer-memory transport (CUDA IPC works within one GPU), and the host-side
    # collectives (barrier, max over ranks, IPC blob exchange) go over gloo,
    # because NCCL refuses two ranks on one device
    ndev = max(1, torch.cuda.device_count())
    shared_gpus = dist_path and world > ndev
    local %= ndev
    torch.cuda.set_device(local)
    coll_dev = "cpu" if shared_gpus else "cuda"
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_maggionibl13_b200 as cme

    comm = None
    replicas = args.replicas and dist_path
    if dist_path:
        if shared_gpus:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        if replicas:
            pass   # independent problems: the process group only carries the timing reductions
        elif args.transport == "nccl":
            obj = [cme.cme_comm_unique_id() if rank == 0 else None]
            dist.broadcast_object_list(obj, src=0)
            comm = cme.cme_comm_init(world, rank, obj[0], local)
        else:
            comm = cme.cme_comm_init_ipc(world, rank, local)

    name = args.config
    B = args.batch
    log("[bench] building", args.config)
    members = replica_members(rank, B) if replicas else list(range(B))
    m, cfg, setup = build_matrix(cme, name, cme.CME_DEVICE_HOST_ONLY if dist_path and not replicas else local, B,
                                 members[0])
    log("[bench] built", setup)
    if comm is not None:
        cme.cme_matrix_distribute(m.h, comm)
        if args.transport == "p2p":
            blobs = [None] * world
            dist.all_gather_object(blobs, cme.cme_matrix_ipc_export(m.h))
            cme.cme_matrix_ipc_attach(m.h, blobs)
    info = m.info()
    n, nnz = info.n, info.nnz
    stream = torch.cuda.Stream()
    m.set_opts(omega=cfg["omega"], check_every=C_BLOCK, stream=stream.cuda_stream)
    cme.cme_solver_load(m.h, n * B, None)
    for _ in range(args.warmup):
        cme.cme_solver_run(m.h, 1)
    torch.cuda.synchronize()

    def barrier():
        if dist_path:
            dist.barrier()
        torch.cuda.synchronize()

    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        barrier()
        e0.record(stream)
        for _ in range(args.steps):
            cme.cme_solver_run(m.h, 1)
        e1.record(stream)
        barrier()
    iters = args.steps * C_BLOCK
    # whole job: max time over ranks; the flops of every rank (a replica run
    # solves world independent problems, a row-sharded one a single matrix)
    ms, work = aggregate(dist, world, coll_dev, e0.elapsed_time(e1), 2.0 * nnz * B * iters)
    if not replicas:
        work = 2.0 * nnz * B * iters
    sec = ms * 1e-3
    gflops = work / sec / 1e9
    peak, peak_src = hbm_peak()
    t_iter = sec / iters
    achieved = info.bytes_alg / t_iter / 1e9        # algorithmic bytes per launch / launch time
    # kernel bytes per iteration: this rank's packed encoding (bytes_fmt is per
    # rank; the whole job moves the sum over ranks in the same time)
    fmt_tot = float(info.bytes_fmt)
    if world > 1:
        tb = torch.tensor([fmt_tot], device=coll_dev, dtype=torch.float64)
        dist.all_reduce(tb, op=dist.ReduceOp.SUM)
        fmt_tot = float(tb.item())
    fmt_gbs = fmt_tot / t_iter / 1e9
    fmt_frac = fmt_gbs / (peak * world)
    enc_bytes = {
        0: "layout v0, 12 B per ELL slot (8 B value + 4 B column) + 8 B inv_d, 4 B row map, 16 B x/y per row",
        1: "compact encoding (DESIGN.md sec. 5b): the rows of M = |D|^-1 O with int16 column and uint8 row "
           "offsets, 10 B per ELL slot + 17 B per row",
        2: "value-indexed compact encoding (DESIGN.md sec. 5c): 16-bit indices into a shared-memory dictionary of "
           "the distinct rates + int16 column offsets (4 B per ELL slot) + inv_d, a uint8 row offset and x/y "
           "(25 B per row)"}[info.compact]
    traffic, traffic_src = ncu_traffic(name, kernel_name(info)) if world == 1 else (None, None)

    log(f"[bench] timed region: {ms / args.steps:.3f} ms/step")
    # e2e: the public solve call with pinned host buffers, H2D + D2H inside the timed region
    p0 = torch.empty(n * B, dtype=torch.float64, pin_memory=True)
    p0.copy_(torch.from_numpy(np.tile(W.uniform_start(n), B)))
    pout = torch.empty(n * B, dtype=torch.float64, pin_memory=True)
    e2e_steps = max(3, min(args.steps, 10))
    cme.cme_jacobi_solve(m.h, n * B, p0, 0.0, C_BLOCK, pout)  # warm
    barrier()
    t = time.perf_counter()
    for _ in range(e2e_steps):
        cme.cme_jacobi_solve(m.h, n * B, p0, 0.0, C_BLOCK, pout)
    barrier()
    e2e_s = time.perf_counter() - t
    if world > 1:
        tt = torch.tensor([e2e_s], device=coll_dev, dtype=torch.float64)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        e2e_s = float(tt.item())
    e2e_gflops = (world if replicas else 1) * 2.0 * nnz * B * C_BLOCK * e2e_steps / e2e_s / 1e9
    clocks = clk.summary()

    # time-to-converge of the benchmark workload itself (BASELINE metric), on
    # every rank of a row-sharded run; device time from the solver's events
    conv_main = None
    if B == 1 and not args.no_converge:
        t = time.perf_counter()
        log("[bench] e2e done; converging", name)
        p_c, st_c, it_c = m.solve(tol=1e-12, max_iter=200000)
        log("[bench] converged", st_c, it_c, "; paper mode")
        wall_c = time.perf_counter() - t
        rep_c = m.report()
        dev_s = rep_c.seconds
        if world > 1:
            tt = torch.tensor([dev_s], device=coll_dev, dtype=torch.float64)
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            dev_s = float(tt.item())
        paper = solve_paper_mode(cme, m, name, cfg["omega"])
        if world > 1:
            tt = torch.tensor([paper["device_seconds"]], device=coll_dev, dtype=torch.float64)
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            paper["device_seconds"] = round(float(tt.item()), 4)
        conv_main = {"workload": name, "tol": 1e-12, "omega": cfg["omega"], "status": st_c, "iters": it_c,
                     "device_seconds": round(dev_s, 4), "wall_seconds": round(wall_c, 4),
                     "delta": rep_c.delta, "mass": float(p_c.sum()),
                     "note": "cme_jacobi_solve from uniform p0; device_seconds = the solve's iteration loop "
                             "(max over ranks), wall includes the p0 load and the D2H of p",
                     "paper_mode": paper}
    conv = None
    if rank == 0 and world == 1 and B == 1 and not args.no_converge:
        try:
            log("[bench] converge_line cfg2")
            conv = converge_line(cme)
        except Exception as ex:  # report, do not hide
            conv = {"error": repr(ex)}
    conv3 = None
    if rank == 0 and world == 1 and B == 1 and not args.no_converge:
        try:
            log("[bench] converge_closed_form cfg3a")
            conv3 = converge_closed_form(cme)
        except Exception as ex:  # report, do not hide
            conv3 = {"error": repr(ex)}
    cpu = None
    if rank == 0 and world == 1 and B == 1 and not args.no_cpu_baseline:
        log("[bench] cpu baseline")
        cb = cpu_oracle_timing(name, budget_s=20.0, omega=cfg["omega"])
        log("[bench] cpu baseline done")
        cpu = {k: cb[k] for k in ("value", "unit", "cores", "kind", "sample", "cpu_model", "value_1thread")}

    if rank == 0:
        line = {
            "metric": "fp64 Jacobi GFLOPS (2 nnz/iteration)", "value": round(gflops, 3), "unit": "GFLOPS",
            "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": round(ms / args.steps, 4), "higher_is_better": True,
            "scaling": "weak" if replicas else "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": (f"{name} sweep, {B} member(s) per rank" if replicas else
                                    name if B == 1 else f"{name} x {B}-member sweep"), "batch": B,
                       "n": n, "nnz": nnz, "order": cfg["order"], "format": "diag_sell",
                       "window": cfg["window"], "band_on": bool(info.band_on), "omega": cfg["omega"],
                       "check_every": C_BLOCK, "iters_per_step": C_BLOCK,
                       "l2": f"inputs larger than L2 ({info.bytes_alg / 1e9:.3f} GB/iteration vs 126 MB)",
                       "parallelism": f"replicas{world}" if replicas else f"rows{world}", "setup": setup,
                       "transport": None if replicas or not dist_path else args.transport},
            "iters_per_s": round(iters / sec, 2),
            "pct_hbm_roofline": round(100.0 * fmt_frac, 2) if fmt_frac is not None else None,
            "roofline": {"bound": "hbm", "achieved": round(fmt_gbs, 1) if fmt_gbs else None,
                         "peak": peak * world, "unit": "GB/s",
                         "frac": round(fmt_frac, 4) if fmt_frac is not None else None,
                         "traffic": traffic, "traffic_source": traffic_src,
                         "peak_source": peak_src, "kernel": kernel_name(info),
                         "bytes_per_launch": info.bytes_fmt,
                         "bytes_note": "the bytes the step kernel must move per iteration for the packed "
                                       "encoding it streams (DESIGN.md sec. 7): " + enc_bytes,
                         "encoding": {0: "layout v0", 1: "compact", 2: "value-indexed compact"}[info.compact],
                         "model_bytes_per_launch": info.bytes_alg,
                         "model_bytes": "12 nnz + 16 n per member (SURVEY 8(d))" if B == 1 else
                                        f"(12 nnz + 16 n) x {B} members: each member counted as if solved alone",
                         "model_gbs": round(achieved, 1),
                         "model_bytes_ratio": round(achieved / (peak * world), 4),
                         "model_note": "SURVEY 8(d) byte model / launch time / peak: > 1 means the encoding moves "
                                       "fewer bytes than the 12 nnz + 16 n model, not a faster-than-HBM kernel",
                         "launch_time_us": round(t_iter * 1e6, 3),
                         "launch_time_note": "timed-region time / step-kernel launches, CUDA events on the "
                                             "solver's stream (includes the 2 tiny check kernels per 100 steps "
                                             "and launch gaps: conservative)"},
            "clocks": clocks,
            "e2e": {"value": round(e2e_gflops, 3), "unit": "GFLOPS", "h2d_bytes_per_step": 8 * n * B,
                    "d2h_bytes_per_step": 8 * n * B, "steps": e2e_steps,
                    "call": "cme_jacobi_solve(h, p0_pinned_host, tol=0, max_iter=100, p_out_pinned_host)"},
            "gpu_launches": args.steps * (C_BLOCK + 2) * 1,
            "time_to_converge": conv_main,
            "converge_paper": {"cfg4": conv_main.get("paper_mode") if conv_main else None,
                               "cfg3a": conv3.get("paper_mode") if isinstance(conv3, dict) else None},
            "converge": conv,
            "converge_closed_form": conv3,
            "cpu_baseline": cpu,
        }
        print(json.dumps(line), flush=True)
    if comm is not None:
        dist.barrier()   # peers may address this rank's buffers until everyone is done
        m.close()
        cme.cme_comm_destroy(comm)
        dist.destroy_process_group()
    elif dist_path:
        dist.barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
