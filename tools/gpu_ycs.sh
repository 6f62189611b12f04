# streaming (evict-first) y stores in the tile-record kernel
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
k() { timeout 900 python tools/kbench.py "$@" 2>&1 | grep "^\[\|rror" | tee -a gpurun_out/ycs_kbench.txt; }
k --config cfg4_toggle_20m --blocks 10 "" "CME_VI2_YCS=1" "" "CME_VI2_YCS=1" "CME_VI2_YCS=1,CME_TMA_XPF=0" "CME_TMA_XPF=0"
k --config banded:16000000:10:1024:0 --blocks 5 "" "CME_VI2_YCS=1"
