# wrap-mode gather with a per-lane select: parity + config 5 width 4096
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
timeout 1500 python -m pytest tests/test_xw.py -q -p no:cacheprovider > gpurun_out/pytest_xw.log 2>&1; tail -3 gpurun_out/pytest_xw.log
export CME_VERBOSE=1
k() { timeout 900 python tools/kbench.py "$@" 2>&1 | grep "^\[\|rror" | grep -v "tma:\|vi2:" | tee -a gpurun_out/wrap2_kbench.txt; }
k --config banded:16000000:10:4096:0 --blocks 5 "" "CME_XW=0"
k --config banded:16000000:10:1024:0 --blocks 5 "" "CME_XW_MODE=2"
k --config banded:16000000:5:8192:0 --blocks 5 "" "CME_XW=0"
