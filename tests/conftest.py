import os

# the workload generator's OpenMP threads must not spin-wait after their parallel regions:
# they would compete for cores with the ctx's host-assist threads (must be set before libgomp loads)
os.environ.setdefault("OMP_WAIT_POLICY", "PASSIVE")
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
