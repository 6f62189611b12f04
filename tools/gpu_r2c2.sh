# full-size config-5 x-window parity, 2-rank row-sharded bench (shared GPU), CPU table with cfg3a converged
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
timeout 1500 python -m pytest tests/test_xw.py -q -p no:cacheprovider --durations=5 > gpurun_out/pytest_xw.log 2>&1; tail -8 gpurun_out/pytest_xw.log
timeout 1200 python bench.py --gpus 2 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_rows2.json 2> gpurun_out/bench_rows2.err; echo "rows2 rc=$?"; head -c 700 gpurun_out/bench_rows2.json; echo
timeout 1500 python tools/cpu_table.py --out gpurun_out/round2_cpu_table --budget 100 > gpurun_out/cpu_table.log 2>&1; tail -4 gpurun_out/cpu_table.log
