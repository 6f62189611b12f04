mkdir -p gpurun_out
timeout 300 python tools/kbench.py --config toggle:400 --blocks 20 CME_RESIDENT=0 CME_RESIDENT=1 2>&1 | grep "^\["
bash tools/gpu_sanitize.sh
timeout 1500 python tools/big_toggle.py --N 7072 > gpurun_out/big_toggle.jsonl 2> gpurun_out/big_toggle.err; tail -1 gpurun_out/big_toggle.jsonl; tail -3 gpurun_out/big_toggle.err
