# x-window kernel: parity, then A/B on cfg4 and config 5
mkdir -p gpurun_out; export CME_VERBOSE=1
python paper_conf_ipps_maggionibl13_b200/build.py
timeout 900 python -m pytest tests/test_xw.py -x -q -p no:cacheprovider > gpurun_out/pytest_xw.log 2>&1; tail -15 gpurun_out/pytest_xw.log
timeout 900 python tools/kbench.py --config cfg4_toggle_20m --blocks 10 "" "CME_XW=1" "CME_XW=1,CME_VI2_WARPS=16" "CME_XW=1,CME_VI2_STAGES=3" 2>&1 | grep "^\[\|rror\|xw" | tee gpurun_out/xw_kbench.txt
timeout 900 python tools/kbench.py --config banded:16000000:10:1024:0 --blocks 5 "" "CME_REC=1" "CME_REC=1,CME_XW=1" "CME_REC=1,CME_XW=1,CME_VI2_WARPS=16" 2>&1 | grep "^\[\|rror\|xw" | tee -a gpurun_out/xw_kbench.txt
timeout 900 python tools/kbench.py --config banded:16000000:10:1024:1 --blocks 5 "" "CME_REC=1,CME_XW=1" "CME_REC=1,CME_XW=1,CME_VI2_WARPS=16" 2>&1 | grep "^\[\|rror\|xw" | tee -a gpurun_out/xw_kbench.txt
timeout 900 python tools/kbench.py --config banded:16000000:10:32:0 --blocks 5 "" "CME_REC=1,CME_XW=1" "CME_REC=1,CME_XW=1,CME_VI2_WARPS=16" 2>&1 | grep "^\[\|rror\|xw" | tee -a gpurun_out/xw_kbench.txt
timeout 900 python tools/kbench.py --config cfg3a_schnakenberg_2m --blocks 10 "" "CME_REC=1,CME_XW=1" "CME_REC=1,CME_XW=1,CME_VI2_WARPS=16" 2>&1 | grep "^\[\|rror\|xw" | tee -a gpurun_out/xw_kbench.txt
