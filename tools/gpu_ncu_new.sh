# ncu full captures of the round-2 kernels not yet profiled: batched records (B = 2) and the wrap-mode x window (width 4096)
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
K1="python tools/kbench.py --config cfg4_toggle_20m --batch 2 --blocks 1 --C 10"
timeout 900 $K1 > gpurun_out/plain_b2.log 2>&1 && \
timeout 1200 ncu --set full --clock-control none -k regex:sell_vi2b -s 20 -c 1 -o gpurun_out/prof_vi2b $K1 > gpurun_out/ncu_b2.log 2>&1; echo "b2 rc=$?"
K2="python tools/kbench.py --config banded:16000000:10:4096:0 --blocks 1 --C 10"
timeout 900 $K2 > gpurun_out/plain_w4k.log 2>&1 && \
timeout 1200 ncu --set full --clock-control none -k regex:sell_vi2 -s 20 -c 1 -o gpurun_out/prof_w4k $K2 > gpurun_out/ncu_w4k.log 2>&1; echo "w4k rc=$?"
