# why widths >= 8192 stay at 60-65%: ncu full capture of the gather kernel on config 5 width 32768 and 8192
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
K="python tools/kbench.py --config banded:16000000:10:32768:0 --blocks 1 --C 10"
timeout 900 $K > gpurun_out/plain_w32k.log 2>&1 && \
timeout 1200 ncu --set full --clock-control none -k regex:"sell_(tma|cpt|vi2)" -s 20 -c 1 -o gpurun_out/prof_w32k $K > gpurun_out/ncu_w32k.log 2>&1; echo "w32k rc=$?"
K2="python tools/kbench.py --config banded:16000000:10:8192:0 --blocks 1 --C 10"
timeout 900 $K2 > gpurun_out/plain_w8k.log 2>&1 && \
timeout 1200 ncu --set full --clock-control none -k regex:"sell_(tma|cpt|vi2)" -s 20 -c 1 -o gpurun_out/prof_w8k $K2 > gpurun_out/ncu_w8k.log 2>&1; echo "w8k rc=$?"
