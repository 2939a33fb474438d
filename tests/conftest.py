"""pytest configuration: the `gpu` marker and shared fixtures.

`-m "not gpu"` runs here (no GPU): oracle pins, host logic, ABI symbol checks,
gloo multi-process tests.  `-m gpu` runs on a B200 through gpurun.
"""
import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA B200 (runs under gpurun)")
    config.addinivalue_line("markers", "slow: long-running case")


@pytest.fixture(scope="session")
def orc():
    import oracle

    oracle.build()
    return oracle


@pytest.fixture(scope="session")
def boidslib():
    """Build (if stale) and load libboids.so -- the CUDA path; no fallback."""
    from paper_conf_ipps_breitbart09_b200 import abi, build

    build.build()
    return abi.load()


def _has_gpu():
    try:
        import torch

        return torch.cuda.is_available()
    except Exception:
        return False


def pytest_collection_modifyitems(config, items):
    if _has_gpu():
        return
    skip = pytest.mark.skip(reason="no CUDA device here (run with -m gpu under gpurun)")
    for it in items:
        if "gpu" in it.keywords:
            it.add_marker(skip)
