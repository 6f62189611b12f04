# x-window kernel: parity + full GPU suite (auto XW now covers small f64 packs), config-5 A/B
mkdir -p gpurun_out
python paper_conf_ipps_maggionibl13_b200/build.py
timeout 900 python -m pytest tests/test_xw.py -q -p no:cacheprovider > gpurun_out/pytest_xw.log 2>&1; tail -5 gpurun_out/pytest_xw.log
timeout 2400 python -m pytest tests -q -m gpu -p no:cacheprovider -x > gpurun_out/pytest_gpu.log 2>&1; tail -5 gpurun_out/pytest_gpu.log
export CME_VERBOSE=1
for cfg in banded:16000000:10:1024:1 banded:16000000:10:4096:0 banded:16000000:5:1024:0 banded:16000000:15:1024:0 banded:100000000:10:1024:0; do
timeout 900 python tools/kbench.py --config $cfg --blocks 5 "CME_XW=0" "" 2>&1 | grep "^\[\|rror" | grep -v "tma:\|vi2:" | tee -a gpurun_out/xw2_kbench.txt
done
timeout 900 python tools/kbench.py --config toggle:1000 --blocks 10 "" "CME_XW=1" 2>&1 | grep "^\[\|rror" | grep -v "tma:\|vi2:" | tee -a gpurun_out/xw2_kbench.txt
