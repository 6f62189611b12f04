#!/usr/bin/env python3
"""CPU oracle timing table ("CPU oracle timing, in the same run on
the same box"): the oracle's plain C CSR Jacobi (oracle/, OpenMP row-parallel,
deterministic blocked sums) on the host cores of the machine it runs on, at 1
thread and at all cores in os.sched_getaffinity(0); cfg1-cfg3a to convergence
(tol 1e-12, C = 100), cfg4 as iterations/s over a bounded sample.  The CPU
model is recorded from /proc/cpuinfo.  Test/measurement infrastructure only
(the oracle is never on the product path).

    python tools/cpu_table.py [--out profiles/round1_cpu_table]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
import workloads as W  # noqa: E402

OMEGA = {"cfg1_birth_death": 0.9, "cfg2_toggle_100k": 0.9, "cfg3a_schnakenberg_2m": 1.0, "cfg4_toggle_20m": 0.9}
# iterations to tol 1e-12 measured on the GPU (same iteration; used only to decide converge vs sample)
EXPECT = {"cfg1_birth_death": 2000, "cfg2_toggle_100k": 3400, "cfg3a_schnakenberg_2m": 44800, "cfg4_toggle_20m": 6400}


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "cpu_table"))
    ap.add_argument("--budget", type=float, default=150.0, help="seconds per converge run before sampling instead")
    a = ap.parse_args()
    cores = len(os.sched_getaffinity(0))
    rows = []
    for name in ("cfg1_birth_death", "cfg2_toggle_100k", "cfg3a_schnakenberg_2m", "cfg4_toggle_20m"):
        A = oracle.network_csr(W.config_network(name))
        om = OMEGA[name]
        for nt in (1, cores):
            t = time.perf_counter()
            oracle.jacobi_solve(A, omega=om, tol=0.0, max_iter=10, stag_tol=0.0, nthreads=nt)
            per = (time.perf_counter() - t) / 10
            row = dict(workload=name, n=A.n, nnz=A.nnz, threads=nt, omega=om)
            if per * EXPECT[name] < a.budget:   # converge if it fits the budget
                t = time.perf_counter()
                r = oracle.jacobi_solve(A, omega=om, tol=1e-12, max_iter=200000, nthreads=nt)
                sec = time.perf_counter() - t
                row.update(mode="to convergence", status=r.status, iters=r.iters, seconds=round(sec, 4),
                           iters_per_s=round(r.iters / sec, 1), gflops=round(2 * A.nnz * r.iters / sec / 1e9, 3))
            else:
                k = max(1, min(100, int(a.budget / 4 / max(per, 1e-9))))
                t = time.perf_counter()
                oracle.jacobi_solve(A, omega=om, tol=0.0, max_iter=k, stag_tol=0.0, nthreads=nt)
                sec = time.perf_counter() - t
                row.update(mode=f"sample of {k} iterations", seconds=round(sec, 3), iters_per_s=round(k / sec, 2),
                           gflops=round(2 * A.nnz * k / sec / 1e9, 3))
            rows.append(row)
            print(json.dumps(row), flush=True)
    info = dict(cpu=cpu_model(), cores=cores, rows=rows)
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    with open(a.out + ".json", "w") as f:
        json.dump(info, f, indent=1)
    with open(a.out + ".md", "w") as f:
        f.write(f"# CPU oracle timing (oracle/ plain C CSR Jacobi, OpenMP) on the GPU box's host\n\n"
                f"CPU: {info['cpu']}, {cores} cores in the affinity mask. fp64, tol 1e-12, C = 100.\n\n"
                "| workload | n | threads | mode | iterations | seconds | iter/s | GFLOPS |\n"
                "|---|---|---|---|---|---|---|---|\n")
        for r in rows:
            f.write(f"| {r['workload']} | {r['n']:,} | {r['threads']} | {r['mode']} | {r.get('iters', '')} | "
                    f"{r['seconds']} | {r['iters_per_s']} | {r['gflops']} |\n")


if __name__ == "__main__":
    main()
