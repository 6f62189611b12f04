# wavefront s-step kernel: parity, then cfg4 timing vs the single-step vi2 kernel; bench phases; L2 probe
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "wavefront" > gpurun_out/wf_pytest.log 2>&1; tail -5 gpurun_out/wf_pytest.log
timeout 900 python tools/kbench.py --config cfg4_toggle_20m --blocks 10 "" "CME_WF=2" "CME_WF=3" "CME_WF=4" "CME_WF=2,CME_WF_KEEP=0" "CME_WF=2,CME_WF_LAG=100" "CME_WF=2,CME_WF_LAG=1000" "CME_WF=4,CME_WF_LAG=800" 2>&1 | grep "^\[\|rror" | tee gpurun_out/wf_kbench.txt
timeout 1200 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -20 gpurun_out/bench.err
bash tools/gpu_l2probe.sh
