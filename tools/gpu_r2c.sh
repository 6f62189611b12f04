# re-entry check of the round-2 state: full GPU suite, smoke, bench, synccheck of the step kernels
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -x -q -m gpu --durations=15 > gpurun_out/pytest_gpu.log 2>&1; tail -25 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; cat gpurun_out/bench.json
CME_RES_TIMEOUT_MS=60000 timeout 1800 compute-sanitizer --tool synccheck --print-limit 20 --error-exitcode 99 python tools/sanitize_case.py > gpurun_out/sanitize_synccheck.log 2>&1
echo "synccheck rc=$?"; tail -4 gpurun_out/sanitize_synccheck.log
