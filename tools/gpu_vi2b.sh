# vi2 shapes: stage depth for the 30-warp CTA, and ncu captures of the 30- and 16-warp kernels on cfg4
mkdir -p gpurun_out
timeout 900 python tools/kbench.py --config cfg4_toggle_20m --blocks 10 "CME_VI2_WARPS=30" "CME_VI2_WARPS=30,CME_VI2_STAGES=5" "CME_VI2_WARPS=30,CME_VI2_STAGES=3" "CME_VI2_WARPS=16,CME_VI2_STAGES=2" 2>&1 | grep "^\["
timeout 600 ncu --set full --import-source on --clock-control none -k regex:sell_vi2 -s 20 -c 1 -o gpurun_out/prof_vi2w30 python tools/kbench.py --config cfg4_toggle_20m --blocks 1 CME_VI2_WARPS=30 > gpurun_out/ncu_vi2w30.log 2>&1; tail -2 gpurun_out/ncu_vi2w30.log
timeout 600 ncu --set full --import-source on --clock-control none -k regex:sell_vi2 -s 20 -c 1 -o gpurun_out/prof_vi2w16 python tools/kbench.py --config cfg4_toggle_20m --blocks 1 CME_VI2_WARPS=16 > gpurun_out/ncu_vi2w16.log 2>&1; tail -2 gpurun_out/ncu_vi2w16.log
