set -x
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m "gpu and not slow" 2>&1 | tail -2
CME_TMA_WARPS=16 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m "gpu and not slow" -k "spmv or landscape" 2>&1 | tail -2
CME_VERBOSE=1 timeout 900 python tools/kbench.py --config cfg4_toggle_20m CME_TMA=0 CME_TMA_STAGES=2 CME_TMA_STAGES=3 CME_TMA_STAGES=2,CME_TMA_CTAS=2 CME_TMA_WARPS=16 CME_TMA_WARPS=16,CME_TMA_STAGES=3 CME_TMA_WARPS=16,CME_TMA_STAGES=4 2>&1
CME_VERBOSE=1 timeout 600 python tools/kbench.py --config cfg3a_schnakenberg_2m CME_TMA=0 CME_TMA_STAGES=2 CME_TMA_STAGES=3 CME_TMA_WARPS=16 CME_TMA_WARPS=16,CME_TMA_STAGES=3 2>&1
