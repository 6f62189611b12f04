# ablation ladder of sell_vi_kernel on cfg4 (CME_ABL levels, kernels_cpt.cuh):
# 1 ring only, 2 + row stream (row8, inv_d, x_r, y), 3 + entry LDS, 4 + own-row loads per entry, 5 + dictionary, base
P=paper_conf_ipps_maggionibl13_b200
mkdir -p gpurun_out
for i in 1 2; do
for v in L1 L2 L3 L4 L5 base; do
  if [ $v = base ]; then L=$PWD/$P/libcme.so; else L=$PWD/$P/libcme_abl_$v.so; fi
  CME_LIBRARY=$L timeout 600 python tools/kbench.py --config cfg4_toggle_20m --blocks 10 "" "CME_TMA_WARPS=31" 2>&1 | grep "^\[" | sed "s/^/$v /"
done
done
