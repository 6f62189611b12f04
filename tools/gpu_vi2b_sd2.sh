mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
export CME_VERBOSE=2
timeout 900 python tools/kbench.py --config cfg4_toggle_20m --batch 2 --blocks 5 "" 2>&1 | grep "vi2b\|^\[default" | tee gpurun_out/vi2b_sd2.txt
