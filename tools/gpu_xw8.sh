# 8-warp x-window tiles (wrap mode) for windows too wide for the 16/30-warp shapes
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
timeout 900 python -m pytest tests/test_xw.py -q -p no:cacheprovider > gpurun_out/pytest_xw.log 2>&1; tail -3 gpurun_out/pytest_xw.log
export CME_VERBOSE=1
k() { timeout 900 python tools/kbench.py "$@" 2>&1 | grep "^\[\|rror" | grep -v "tma:\|vi2:" | tee -a gpurun_out/xw8_kbench.txt; }
k --config banded:16000000:10:8192:0 --blocks 5 "CME_XW=0" "CME_XW=1" "CME_XW=1,CME_VI2_STAGES=2"
k --config banded:16000000:10:4096:0 --blocks 5 "" "CME_XW=1,CME_VI2_WARPS=8"
k --config banded:16000000:5:8192:0 --blocks 5 "CME_XW=0" "CME_XW=1"
k --config banded:16000000:15:8192:1 --blocks 5 "CME_XW=0" "CME_XW=1"
k --config banded:16000000:10:16384:0 --blocks 5 "CME_XW=0" "CME_XW=1"
