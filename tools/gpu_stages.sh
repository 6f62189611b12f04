mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
export CME_VERBOSE=1
timeout 900 python tools/kbench.py --config cfg4_toggle_20m --blocks 10 "" "CME_VI2_STAGES=5" "CME_VI2_STAGES=6" "" "CME_VI2_STAGES=5" 2>&1 | grep "vi2:\|^\[default\|^\[CME" | tee gpurun_out/stages_kbench.txt
