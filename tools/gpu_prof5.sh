mkdir -p gpurun_out
for w in 1024 32 32768; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sell_tma -s 50 -c 1 -o gpurun_out/prof_cfg5_w$w python tools/kbench.py --config banded:16000000:10:$w:0 --blocks 1 > gpurun_out/ncu_cfg5_w$w.log 2>&1
tail -2 gpurun_out/ncu_cfg5_w$w.log
done
ls -la gpurun_out
