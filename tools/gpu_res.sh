mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "every_step_kernel or resident or landscape or closed or spmv or stagnation or residual or max_iter or device_pointers or invalid" > gpurun_out/pytest_res.log 2>&1; tail -15 gpurun_out/pytest_res.log
CME_VERBOSE=1 timeout 300 python tools/kbench.py --config cfg2_toggle_100k --blocks 30 CME_RESIDENT=0 CME_RESIDENT=1 2>&1 | grep -v "^enumerated" | tail -8
timeout 300 python tools/kbench.py --config cfg1_birth_death --blocks 30 CME_RESIDENT=0 CME_RESIDENT=1 2>&1 | tail -3
timeout 300 python bench.py --config cfg2_toggle_100k --steps 10 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['converge'])"
