mkdir -p gpurun_out
free -g | head -2; nproc
timeout 300 python tools/kbench.py --config toggle:400 --blocks 20 CME_RESIDENT=0 CME_RESIDENT=1 2>&1 | tail -2
timeout 300 python tools/kbench.py --config toggle:300 --blocks 20 CME_RESIDENT=0 CME_RESIDENT=1 2>&1 | tail -2
timeout 2400 python tools/sweep_cfg5.py --out gpurun_out/cfg5_sweep 2>&1 | tail -30
