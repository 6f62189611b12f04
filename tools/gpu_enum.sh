timeout 900 python -m pytest tests/test_gpu_enumerate.py -x -q -s 2>&1 | tail -15
timeout 600 python -c "
import time, workloads as W, paper_conf_ipps_maggionibl13_b200 as cme
for N in (224, 1000, 3164):
    net = W.toggle_switch(N)
    t=time.perf_counter(); g=cme.cme_network_enumerate_gpu(net); tg=time.perf_counter()-t
    t=time.perf_counter(); h=cme.cme_network_enumerate(net); th=time.perf_counter()-t
    print(f'toggle N={N}: n={len(g[0])} gpu {tg:.3f}s host(DFS) {th:.3f}s')
net = W.schnakenberg(2000)
t=time.perf_counter(); g=cme.cme_network_enumerate_gpu(net); tg=time.perf_counter()-t
t=time.perf_counter(); h=cme.cme_network_enumerate(net); th=time.perf_counter()-t
print(f'schnakenberg N=2000: n={len(g[0])} gpu {tg:.3f}s host(DFS) {th:.3f}s')
"
