# contiguous tile ranges for the gather kernel (L1 reuse of the x band across consecutive tiles)
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
k() { timeout 900 python tools/kbench.py "$@" 2>&1 | grep "^\[\|rror" | tee -a gpurun_out/contig_kbench.txt; }
k --config cfg4_toggle_20m --blocks 10 "" "CME_VI2_CONTIG=1" "CME_VI2_CONTIG=1,CME_VI2_STAGES=3" "CME_VI2_CONTIG=1,CME_VI2_STAGES=2" "CME_VI2_CONTIG=1,CME_VI2_WARPS=16,CME_VI2_STAGES=2" ""
k --config toggle:2200 --blocks 10 "" "CME_VI2_CONTIG=1" "CME_VI2_CONTIG=1,CME_VI2_STAGES=2"
