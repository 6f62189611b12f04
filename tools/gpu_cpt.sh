mkdir -p gpurun_out
for cfg in cfg3a_schnakenberg_2m cfg4_toggle_20m; do
timeout 600 python tools/kbench.py --config $cfg --blocks 10 CME_COMPACT=0 CME_VI=0 CME_VI=0,CME_TMA_XPF=1 CME_VI=0,CME_TMA_STAGES=2 CME_VI=1 2>&1 | grep "^\["
done
