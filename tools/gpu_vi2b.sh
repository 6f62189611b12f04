# batched tile records (sell_vi2b_kernel): parity, then cfg4 B = 2/4/8 against sell_vib_kernel
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
timeout 1500 python -m pytest tests/test_batch.py -q -p no:cacheprovider -x > gpurun_out/pytest_batch.log 2>&1; tail -3 gpurun_out/pytest_batch.log
export CME_VERBOSE=1
for b in 2 4 8; do timeout 900 python tools/kbench.py --config cfg4_toggle_20m --batch $b --blocks 5 "CME_VI2B=0" "" "CME_VI2_WARPS=$( [ $b = 2 ] && echo 16 || ( [ $b = 4 ] && echo 30 || echo 8 ) )" 2>&1 | grep "^\[\|rror" | grep -v "tma:" | tee -a gpurun_out/vi2b_kbench.txt; done
