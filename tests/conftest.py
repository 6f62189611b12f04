import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

# Virtual-rank groups (test_p2p_group.py) run up to 8 ranks in this process,
# each with its own streams; with the default 8 hardware work queues the
# streams alias, and one rank's spinning flag-barrier / gated step kernel
# then blocks the queue a peer's kernel sits behind (observed: 8-rank groups
# time out).  Must be set before the CUDA context exists.
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: multi-second CPU test")


@pytest.fixture(scope="session")
def oracle_mod():
    import oracle
    oracle.build()
    return oracle
