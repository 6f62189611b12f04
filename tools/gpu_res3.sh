mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "resident or every_step or landscape or spmv" 2>&1 | tail -3
CME_VERBOSE=1 timeout 300 python tools/kbench.py --config cfg2_toggle_100k --blocks 30 CME_RESIDENT=1 2>&1 | grep "^\[" 
timeout 300 python tools/kbench.py --config toggle:300 --blocks 20 CME_RESIDENT=1 2>&1 | grep "^\["
bash tools/gpu_sanitize.sh
