import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")


@pytest.fixture(scope="session")
def c1_mesh():
    import gen
    return gen.kuhn_duct(6, 6, 30)


@pytest.fixture(scope="session")
def c1_mesh_jit():
    import gen
    return gen.kuhn_duct(6, 6, 30, jitter=0.2, seed=7)
