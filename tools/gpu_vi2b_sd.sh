# B = 2 batched records with the tuple dictionary staged in shared memory
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
timeout 1500 python -m pytest tests/test_batch.py -q -p no:cacheprovider > gpurun_out/pytest_batch.log 2>&1; tail -2 gpurun_out/pytest_batch.log
export CME_VERBOSE=1
timeout 900 python tools/kbench.py --config cfg4_toggle_20m --batch 2 --blocks 10 "CME_VI2B=0" "CME_VI2B_SD=0" "" "CME_VI2B_SD=0" "" 2>&1 | grep "^\[\|rror" | grep -v "tma:" | tee gpurun_out/vi2b_sd_kbench.txt
