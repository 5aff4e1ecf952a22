import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (sm_100a) and the built libqoserve.so")
    config.addinivalue_line("markers", "slow: long-running CPU test")


def _has_gpu():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


@pytest.fixture(scope="session")
def gpu_available():
    return _has_gpu()


def pytest_collection_modifyitems(config, items):
    # GPU tests are never silently skipped on a GPU box; without a GPU they are skipped
    # only when the caller did not explicitly select them with -m gpu.
    if _has_gpu():
        return
    markexpr = config.getoption("-m") or ""
    if markexpr.strip() == "gpu":
        return  # let them fail loudly: someone asked for GPU tests on a CPU box
    skip = pytest.mark.skip(reason="no CUDA device")
    for it in items:
        if "gpu" in it.keywords:
            it.add_marker(skip)
