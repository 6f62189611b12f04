# round-2 measurement session A (no ncu): GPU suite, smoke, bench (both arms), config-5 sweep, CPU table
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
timeout 2400 python -m pytest tests -q -m gpu -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; tail -4 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; head -c 400 gpurun_out/bench.json; echo
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err; head -c 300 gpurun_out/bench_ref.json; echo
timeout 2400 python tools/sweep_cfg5.py --out gpurun_out/round2_cfg5_sweep > gpurun_out/sweep.log 2>&1; tail -3 gpurun_out/sweep.log
timeout 1500 python tools/cpu_table.py --out gpurun_out/round2_cpu_table --budget 60 > gpurun_out/cpu_table.log 2>&1; tail -3 gpurun_out/cpu_table.log
