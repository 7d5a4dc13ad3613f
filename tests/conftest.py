import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running (large n)")


@pytest.fixture(scope="session")
def rng():
    import numpy as np
    return np.random.default_rng(12345)

# Specialise (NVRTC) only passes of >= 2^20 amplitudes in the test suite, to keep its compile
# time bounded; the JIT path itself is covered by the jit=2 tests and the full-size tests.
os.environ.setdefault("QGPU_JIT_MIN_BITS", "20")
