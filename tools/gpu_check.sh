set -x
timeout 900 python tools/kbench.py --config cfg4_toggle_20m CME_TMA=1 CME_TMA=1 2>&1
timeout 600 python tools/kbench.py --config cfg3a_schnakenberg_2m CME_TMA=1 2>&1
