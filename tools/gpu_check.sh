set -x
timeout 900 python -m pytest tests/test_p2p_group.py -x -q 2>&1 | tail -15
