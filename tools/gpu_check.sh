set -x
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m "gpu" 2>&1 | tail -4
CME_VERBOSE=1 timeout 600 python tools/kbench.py --config cfg2_toggle_100k --blocks 50 CME_TMA=0,CME_PERSIST=0 CME_PERSIST=1 CME_TMA=1 2>&1
timeout 600 python tools/kbench.py --config cfg3a_schnakenberg_2m CME_PERSIST=1 CME_TMA=0,CME_PERSIST=0 CME_TMA=1 2>&1
timeout 600 python tools/kbench.py --config banded:1000000:10:64:1 --blocks 20 CME_PERSIST=1 CME_TMA=0,CME_PERSIST=0 CME_TMA=1 2>&1
