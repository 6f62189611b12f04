# 31 consumer warps (1024-thread CTA) for the cfg4 tile-record kernel
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
export CME_VERBOSE=1
k() { timeout 900 python tools/kbench.py "$@" 2>&1 | grep "^\[\|rror" | grep -v "tma:" | tee -a gpurun_out/w31_kbench.txt; }
k --config cfg4_toggle_20m --blocks 10 "" "CME_VI2_WARPS=31" "" "CME_VI2_WARPS=31" "CME_VI2_WARPS=31,CME_VI2_STAGES=3"
timeout 600 python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -k "vi2_ring_wraps or value_index_bit_identical" > gpurun_out/pytest_w31.log 2>&1; tail -2 gpurun_out/pytest_w31.log
