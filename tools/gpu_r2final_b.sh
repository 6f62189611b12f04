# round-2 measurement session B (ncu): launch list of the bench, full captures of the two hot kernels,
# plus ordering experiments on cfg4 (no ncu)
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
timeout 900 python tools/kbench.py --config cfg4_toggle_20m --order dfs --blocks 10 "" 2>&1 | grep "^\[\|rror" | tee gpurun_out/order_kbench.txt
timeout 900 python tools/kbench.py --config cfg4_toggle_20m --blocks 10 "" "CME_VI2_WORDS=1" 2>&1 | grep "^\[\|rror" | tee -a gpurun_out/order_kbench.txt
B="python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-converge"
timeout 900 $B > gpurun_out/plain_bench.log 2>&1 && \
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 420 --csv --log-file gpurun_out/round2_cfg4_launches.csv $B > gpurun_out/ncu_launch_bench.log 2>&1; echo "launch list rc=$?"
K4="python tools/kbench.py --config cfg4_toggle_20m --blocks 1 --C 10"
timeout 900 $K4 > gpurun_out/plain_k4.log 2>&1 && \
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:sell_vi2 -s 20 -c 2 -o gpurun_out/prof_cfg4_vi2 $K4 > gpurun_out/ncu_k4.log 2>&1; echo "cfg4 full rc=$?"
K5="python tools/kbench.py --config banded:16000000:10:1024:0 --blocks 1 --C 10"
timeout 900 $K5 > gpurun_out/plain_k5.log 2>&1 && \
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:sell_vi2 -s 20 -c 2 -o gpurun_out/prof_cfg5_xw $K5 > gpurun_out/ncu_k5.log 2>&1; echo "cfg5 full rc=$?"
timeout 900 python bench.py --gpus 2 --replicas --steps 5 --warmup 3 --no-cpu-baseline --no-converge > gpurun_out/bench_replicas2.json 2> gpurun_out/bench_replicas2.err; echo "replicas rc=$?"; head -c 600 gpurun_out/bench_replicas2.json
ls -la gpurun_out
