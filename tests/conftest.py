"""Shared test setup. Markers: `gpu` = needs a CUDA device (run on the B200 box)."""
import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); run with -m gpu")
    config.addinivalue_line("markers", "slow: full-size configs (minutes)")


@pytest.fixture(scope="session", autouse=True)
def _built():
    """Build the oracle and the native libraries in-tree once per session (no-op when fresh)."""
    import oracle
    from paper_conf_isca_stephensonhlejn15_b200 import _build
    oracle.build()
    _build.build()
    yield
