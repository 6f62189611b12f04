# packed vidx|col16 words (one LDS per entry): parity, then interleaved A/B against the previous build on cfg4
mkdir -p gpurun_out
P=paper_conf_ipps_maggionibl13_b200
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_p2p_group.py tests/test_batch.py -x -q -m gpu > gpurun_out/pytest_vc.log 2>&1; tail -3 gpurun_out/pytest_vc.log
for i in 1 2; do
  timeout 600 python tools/kbench.py --config cfg4_toggle_20m --blocks 10 "" 2>&1 | grep "^\[" | sed 's/^/new  /'
  CME_LIBRARY=$PWD/$P/libcme_prev.so timeout 600 python tools/kbench.py --config cfg4_toggle_20m --blocks 10 "" 2>&1 | grep "^\[" | sed 's/^/prev /'
done
