"""pytest configuration: registers the ``gpu`` marker and builds the host-side
native libraries (generators, oracle, and — when nvcc is present — libefg.so)."""
import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA B200 (run with -m gpu)")
    config.addinivalue_line("markers", "slow: full-size (BASELINE.json) parity cases")
    import __graft_entry__ as ge
    ge.build_host()
    if os.path.exists(ge.NVCC) and ge.product_sources():
        ge.build_product()


@pytest.fixture(scope="session")
def cuda_ok():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("test marked gpu but no CUDA device is visible")
    return True
