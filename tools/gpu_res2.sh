P=paper_conf_ipps_maggionibl13_b200
for lib in libcme.so libcme_ldcg.so libcme_ldvol.so libcme_noprobe.so; do
  CME_LIBRARY=$PWD/$P/$lib timeout 300 python tools/kbench.py --config cfg2_toggle_100k --blocks 30 CME_RESIDENT=1 2>&1 | grep "^\[" | sed "s/^/$lib /"
  CME_LIBRARY=$PWD/$P/$lib timeout 300 python tools/kbench.py --config cfg1_birth_death --blocks 30 CME_RESIDENT=1 2>&1 | grep "^\[" | sed "s/^/$lib /"
done
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sell_resident -c 1 -o gpurun_out/prof_res python tools/kbench.py --config cfg2_toggle_100k --blocks 5 CME_RESIDENT=1 > gpurun_out/ncu_res.log 2>&1; tail -2 gpurun_out/ncu_res.log
timeout 1200 python - <<'PY'
import time, numpy as np, workloads as W, paper_conf_ipps_maggionibl13_b200 as cme
net = W.config_network("cfg4_toggle_20m")
t = time.perf_counter()
m = cme.Matrix.from_network(net, gpu=True).reorder(cme.CME_ORDER_RCM).pack()
print(f"setup (gpu enumerate + ingest + rcm + pack) {time.perf_counter()-t:.1f}s", flush=True)
m.set_opts(omega=0.9, check_every=100)
p, st, it = m.solve(tol=1e-12, max_iter=3_000_000)
rep = m.report()
print(f"cfg4 converge: status={st} iters={it} device_s={rep.seconds:.2f} delta={rep.delta:.3e} resid={rep.resid:.3e} mass={p.sum():.15f}", flush=True)
S = m.states
onoff = p[(S[:, 0] > S[:, 1])].sum()
print(f"mass with pA > pB: {onoff:.6f}; max p {p.max():.3e}", flush=True)
np.save("gpurun_out/cfg4_landscape_head.npy", p[:1000])
PY
