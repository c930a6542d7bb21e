"""pytest configuration: the ``gpu`` marker (tests that need a B200 and the built CUDA library)."""
import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a) and the built libstarsim.so")
    config.addinivalue_line("markers", "slow: full-size parity case (minutes of oracle time)")
