timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_p2p_group.py -x -q -m gpu 2>&1 | tail -1
timeout 600 python tools/kbench.py --config cfg4_toggle_20m --blocks 10 CME_VI=1 CME_VI=0 2>&1 | grep "^\["
