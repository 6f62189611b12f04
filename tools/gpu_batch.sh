# batched value-indexed kernel (sell_vib_kernel) on cfg4: B = 2, 4, 8
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
for b in 2 4 8; do timeout 900 python tools/kbench.py --config cfg4_toggle_20m --batch $b --blocks 5 "" 2>&1 | grep "^\[\|rror" | tee -a gpurun_out/batch_kbench.txt; done
