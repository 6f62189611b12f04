timeout 900 python -m pytest tests/test_batch.py -x -q -m gpu 2>&1 | grep -E "^E |FAILED|passed|failed" | head -8
for b in 2 4 8; do CME_VERBOSE=1 timeout 900 python tools/kbench.py --config cfg4_toggle_20m --batch $b --blocks 5 CME_VI=0 CME_VI=1 2>&1 | grep "^\[" | grep -v "compact=0 vi=0"; done
