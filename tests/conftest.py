import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); parity tests through the C-ABI")
    config.addinivalue_line("markers", "slow: long CPU test")
    config.addinivalue_line("markers", "scale27: R-MAT scale-27 (C5) GPU parity, ~120 GB device memory")


SEEDS = (1, 42, 2**64 - 1)   # method seeds swept for parity
