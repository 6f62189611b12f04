set -x
timeout 1500 python -m pytest tests -x -q -m "gpu and not slow" 2>&1 | tail -2
timeout 900 python tools/kbench.py --config cfg4_toggle_20m --blocks 20 CME_TMA=1 CME_TMA=1 2>&1
timeout 600 python tools/kbench.py --config cfg3a_schnakenberg_2m CME_TMA=1 2>&1
