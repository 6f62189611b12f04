# full GPU suite (no -x: see every failure), smoke, kernel experiments, bench
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
timeout 2400 python -m pytest tests -q -m gpu -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; tail -15 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout 900 python tools/kbench.py --config cfg4_toggle_20m --blocks 10 "" "CME_VI2_STAGES=2" "CME_VI2_STAGES=3" "CME_VI2_WARPS=16" 2>&1 | grep "^\[\|rror" | tee gpurun_out/r2b_kbench.txt
timeout 900 python tools/kbench.py --config cfg4_toggle_20m --window 1 --blocks 10 "" "CME_VI2_STAGES=2" 2>&1 | grep "^\[\|rror" | tee -a gpurun_out/r2b_kbench.txt
timeout 900 python tools/kbench.py --config cfg3a_schnakenberg_2m --blocks 10 "CME_REC=0" "" "CME_VI2_WARPS=16" 2>&1 | grep "^\[\|rror" | tee -a gpurun_out/r2b_kbench.txt
timeout 900 python tools/kbench.py --config banded:16000000:10:1024:0 --blocks 5 "CME_REC=0" "" "CME_VI2_WARPS=16" 2>&1 | grep "^\[\|rror" | tee -a gpurun_out/r2b_kbench.txt
timeout 1200 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -12 gpurun_out/bench.err; head -c 600 gpurun_out/bench.json
