# the 100M-state toggle (N = 7072) on the round-2 kernels: GPU enumeration, RCM, tile records, solve to 1e-12
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
CME_VERBOSE=1 timeout 1800 python tools/big_toggle.py --N 7072 > gpurun_out/big_toggle.jsonl 2> gpurun_out/big_toggle.err; tail -1 gpurun_out/big_toggle.jsonl; grep "vi2\|tma:" gpurun_out/big_toggle.err | tail -3; tail -3 gpurun_out/big_toggle.err
