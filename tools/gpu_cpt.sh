# compact encoding / x prefetch A/B on the bench workloads
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "compact or every_step or transient" > gpurun_out/pytest_cpt.log 2>&1; tail -3 gpurun_out/pytest_cpt.log
for cfg in cfg4_toggle_20m cfg3a_schnakenberg_2m banded:16000000:10:1024:0 banded:16000000:10:32:0; do
  timeout 600 python tools/kbench.py --config $cfg --blocks 10 CME_COMPACT=0,CME_TMA_XPF=0 CME_COMPACT=0,CME_TMA_XPF=1 CME_COMPACT=1,CME_TMA_XPF=0 CME_COMPACT=1,CME_TMA_XPF=1 CME_COMPACT=1,CME_TMA_XPF=1,CME_TMA_STAGES=3 CME_COMPACT=1,CME_TMA_XPF=1,CME_TMA_WARPS=8,CME_TMA_STAGES=3 2>&1 | grep "^\["
done
