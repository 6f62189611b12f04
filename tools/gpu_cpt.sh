mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "compact or every_step or transient or value_index" > gpurun_out/pyt.log 2>&1; tail -2 gpurun_out/pyt.log; grep -B3 "^E " gpurun_out/pyt.log | head -30
for cfg in cfg4_toggle_20m; do
CME_VERBOSE=2 timeout 600 python tools/kbench.py --config $cfg --blocks 10 CME_VI=1,CME_TMA_SPW=1 CME_VI=1,CME_TMA_SPW=2 CME_VI=1,CME_TMA_SPW=2,CME_TMA_STAGES=3 2>&1 | grep "^\[" | grep -v "compact=0\|extra=0"
done
