# final config-5 sweep with the current x-window kernels
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
timeout 2400 python tools/sweep_cfg5.py --out gpurun_out/round2_cfg5_sweep > gpurun_out/sweep.log 2>&1; tail -3 gpurun_out/sweep.log
