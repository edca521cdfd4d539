import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); run with -m gpu")
    config.addinivalue_line("markers", "slow: full-size oracle work (seconds to minutes)")


@pytest.fixture(scope="session")
def cfg1_grid():
    import synthgrid
    return synthgrid.make_config(1)


@pytest.fixture(scope="session")
def cfg1_oracle(cfg1_grid):
    import oracle
    return oracle.grid(cfg1_grid.tiles)
