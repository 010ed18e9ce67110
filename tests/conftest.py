import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA B200 (runs the sm_100a kernels through the C-ABI)")
    config.addinivalue_line("markers", "slow: larger CPU cases")


@pytest.fixture(scope="session")
def tiny():
    import forestgen
    return forestgen.generate("tiny")


@pytest.fixture(scope="session")
def c1e4():
    import forestgen
    return forestgen.generate("c1e4")


@pytest.fixture(scope="session", params=["tiny", "tiny_c"])
def tinyx(request):
    """tiny, and tiny with C-shape detours (row f4, reading Q14b)"""
    import forestgen
    return forestgen.generate(request.param)
