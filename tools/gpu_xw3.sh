# exact-size x ring: parity, then where XW pays (config 5 widths, cfg3a, toggles)
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
timeout 900 python -m pytest tests/test_xw.py -q -p no:cacheprovider > gpurun_out/pytest_xw.log 2>&1; tail -3 gpurun_out/pytest_xw.log
export CME_VERBOSE=1
k() { timeout 900 python tools/kbench.py "$@" 2>&1 | grep "^\[\|rror" | grep -v "tma:\|vi2:" | tee -a gpurun_out/xw3_kbench.txt; }
k --config banded:16000000:10:1024:0 --blocks 5 "CME_XW=0" ""
k --config banded:16000000:10:4096:0 --blocks 5 "CME_XW=0" "" "CME_XW=1"
k --config banded:16000000:10:8192:0 --blocks 5 "CME_XW=0" "CME_XW=1"
k --config banded:16000000:10:4096:1 --blocks 5 "CME_XW=0" ""
k --config cfg3a_schnakenberg_2m --blocks 10 "CME_XW=0" "" "CME_XW=1"
k --config toggle:1000 --blocks 10 "" "CME_XW=1"
k --config cfg4_toggle_20m --blocks 10 "" "CME_XW=1"
