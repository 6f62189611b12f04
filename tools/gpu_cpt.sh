for cfg in cfg4_toggle_20m cfg3a_schnakenberg_2m banded:16000000:10:32768:0 banded:16000000:5:1024:0 banded:4000000:10:1024:0; do
CME_VERBOSE=1 timeout 600 python tools/kbench.py --config $cfg --blocks 5 CME_VI=1 CME_VI=0 2>&1 | grep "^\[" | grep -v "^\[cme\]"
done
