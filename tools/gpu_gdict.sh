# x window with the value index's dictionary in global memory (ENC 3): parity, cfg4 A/B
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
timeout 1500 python -m pytest tests/test_xw.py -q -p no:cacheprovider -k "not full_size" > gpurun_out/pytest_xw.log 2>&1; tail -3 gpurun_out/pytest_xw.log
export CME_VERBOSE=1
k() { timeout 900 python tools/kbench.py "$@" 2>&1 | grep "^\[\|rror" | grep -v "tma:\|vi2:" | tee -a gpurun_out/gdict_kbench.txt; }
k --config cfg4_toggle_20m --blocks 10 "" "CME_XW=1,CME_XW_GDICT=1" "CME_XW=1,CME_XW_GDICT=1,CME_VI2_STAGES=2" "CME_XW=1,CME_XW_GDICT=1,CME_VI2_WARPS=16"
k --config toggle:2200 --blocks 10 "" "CME_XW=1,CME_XW_GDICT=1" "CME_XW=1,CME_XW_GDICT=1,CME_VI2_STAGES=2"
