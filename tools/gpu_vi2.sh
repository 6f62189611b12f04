# tile-record value-indexed kernel: parity subset, then cfg4 A/B (packed words, shapes)
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "vi2 or every_step or compact_tma or value_index or signed or transient or ablation" > gpurun_out/vi2_pytest.log 2>&1; tail -3 gpurun_out/vi2_pytest.log
for i in 1 2; do
timeout 900 python tools/kbench.py --config cfg4_toggle_20m --blocks 10 "" "CME_VI2_WORDS=1" "CME_VI2_WARPS=16" "CME_VI2_WARPS=16,CME_VI2_WORDS=1" "CME_VI2=0" 2>&1 | grep "^\["
done
