import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    # a fresh checkout has no built artefacts: compile libstg.so (nvcc cross-compiles
    # sm_100a without a GPU) and the C oracle before any test module imports them
    import __graft_entry__
    __graft_entry__.build()
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: large inputs (full-size configs)")


@pytest.fixture(scope="session")
def stg():
    """The CUDA product library through its Python binding (fails loudly if missing)."""
    import paper_conf_ipps_cherianmcc24_b200 as m
    return m
