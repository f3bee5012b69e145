import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (runs through the CUDA C-ABI path)")
    config.addinivalue_line("markers", "slow: long-running CPU test")


def pytest_collection_modifyitems(config, items):
    # GPU tests fail loudly (never skip silently) when selected without a GPU;
    # they are deselected by -m "not gpu" on the CPU box.
    pass


@pytest.fixture(scope="session")
def golden():
    import json

    d = os.path.join(os.path.dirname(__file__), "golden")

    def load(name):
        with open(os.path.join(d, name)) as f:
            return json.load(f)
    return load
