# fused in-kernel halo sync: virtual-rank and IPC groups
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
timeout 1200 python -m pytest tests/test_p2p_group.py tests/test_ipc_group.py -q -m gpu -p no:cacheprovider --durations=12 > gpurun_out/fused_pytest.log 2>&1; tail -25 gpurun_out/fused_pytest.log
