import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); run with -m gpu")
    config.addinivalue_line("markers", "slow: long-running CPU pin")


@pytest.fixture(scope="session", autouse=True)
def _native_build():
    """Build every in-tree native artefact once per session (make is incremental)."""
    subprocess.check_call(["make", "-s", "-C", ROOT, "all"])
    yield
