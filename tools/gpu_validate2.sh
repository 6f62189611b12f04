# final validation: full GPU suite, smoke, bench, and every kernel variant once (sanitize_case.py without the sanitizer)
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
timeout 600 python tools/sanitize_case.py > gpurun_out/kernel_variants.log 2>&1; echo "variants rc=$?"; tail -3 gpurun_out/kernel_variants.log
timeout 2400 python -m pytest tests -q -m gpu -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; tail -2 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; head -c 200 gpurun_out/bench.json; echo
