import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (runs through the C-ABI library)")
    config.addinivalue_line("markers", "slow: oracle checks at Set-B size (tens of seconds)")


@pytest.fixture(scope="session", autouse=True)
def _oracle_built():
    from oracle import build
    build()
