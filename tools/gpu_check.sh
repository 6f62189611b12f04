set -x
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -x -q -m "gpu" > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
timeout 300 python tools/kbench.py --config cfg1_birth_death --blocks 100 CME_PERSIST=0 CME_PERSIST=1 2>&1
timeout 1800 python tools/ablation.py --out gpurun_out/ablation.json > gpurun_out/ablation.log 2>&1; tail -45 gpurun_out/ablation.log
