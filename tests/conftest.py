import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: large inputs (full-size configs)")


@pytest.fixture(scope="session")
def stg():
    """The CUDA product library through its Python binding (fails loudly if missing)."""
    import paper_conf_ipps_cherianmcc24_b200 as m
    return m
