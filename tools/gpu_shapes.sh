# tile-shape experiments: parity of the new shapes, then cfg4 timings (batches 16 vs 15 consumer warps)
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_batch.py -x -q -m gpu -k "bit_identical or every_step_kernel or batch_spmv" > gpurun_out/pytest_shapes.log 2>&1; tail -3 gpurun_out/pytest_shapes.log
for B in 4 8 2; do
  CME_VERBOSE=2 timeout 900 python tools/kbench.py --config cfg4_toggle_20m --batch $B --blocks 5 CME_TMA_WARPS=16 CME_TMA_WARPS=15 2>&1 | grep "^\[CME\|tma:"
done
