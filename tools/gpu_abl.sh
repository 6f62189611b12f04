# ablations of sell_vi_kernel on cfg4: which part of the consumer loop sets the time
P=paper_conf_ipps_maggionibl13_b200
mkdir -p gpurun_out
for i in 1 2; do
for v in base NOINVD STREAM; do
  if [ $v = base ]; then L=$PWD/$P/libcme.so; else L=$PWD/$P/libcme_abl_$v.so; fi
  CME_LIBRARY=$L timeout 600 python tools/kbench.py --config cfg4_toggle_20m --blocks 10 "CME_VI_IDPF=0" "CME_VI_IDPF=1" "CME_TMA_WARPS=31,CME_VI_IDPF=1" "CME_TMA_WARPS=31,CME_VI_IDPF=1,CME_TMA_STAGES=6" 2>&1 | grep "^\[" | sed "s/^/$v /"
done
done
