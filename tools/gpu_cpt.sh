for i in 1 2 3; do timeout 900 python -m pytest tests/test_p2p_group.py tests/test_ipc_group.py -x -q -m gpu 2>&1 | tail -1; done
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_batch.py -x -q -m gpu 2>&1 | tail -1
