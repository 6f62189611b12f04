mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2base_smi.txt
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/r2base_pytest.log 2>&1; tail -3 gpurun_out/r2base_pytest.log
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/r2base_bench.json 2> gpurun_out/r2base_bench.err; tail -c 600 gpurun_out/r2base_bench.json
