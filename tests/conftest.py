import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (runs the CUDA path through the C-ABI)")
    config.addinivalue_line("markers", "slow: full-size configurations")
    # Build the native libraries once per session (incremental; nvcc cross-compiles on CPU).
    sys.path.insert(0, os.path.join(ROOT, "tools"))
    import build  # noqa: E402
    build.build_all()


def cuda_ok() -> bool:
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


@pytest.fixture(scope="session")
def karate():
    import graphgen
    return graphgen.karate()
