mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
timeout 2400 python tools/ablation.py --out gpurun_out/round2_ablation.json > gpurun_out/ablation.log 2>&1; tail -2 gpurun_out/ablation.log
