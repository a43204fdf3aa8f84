import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running CPU test")


@pytest.fixture(scope="session")
def inputs_cache():
    """Session cache of nasgen inputs keyed by (nx, ny, nz, seed, A, B, dt)."""
    import nasgen
    cache = {}

    def get(nx, ny=None, nz=None, seed=1, A=1e-3, B=0.0, dt=0.001):
        ny = nx if ny is None else ny
        nz = nx if nz is None else nz
        key = (nx, ny, nz, seed, A, B, dt)
        if key not in cache:
            cache[key] = nasgen.make_inputs(nx, ny, nz, seed=seed, A=A, B=B, dt=dt)
        return cache[key]

    return get
