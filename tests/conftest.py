import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (CUDA) and the built libgist.so")
    config.addinivalue_line("markers", "slow: long-running (exhaustive sweeps)")


@pytest.fixture(scope="session")
def ref():
    import oracle
    oracle.lib()
    return oracle


@pytest.fixture(scope="session")
def gist():
    """The product package (CUDA path).  Builds libgist.so in-tree if needed (nvcc
    cross-compiles without a GPU)."""
    import build_gist
    build_gist.build()
    import paper_conf_isca_jainpmtp18_b200 as g
    return g


@pytest.fixture(scope="session")
def cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    return torch.device("cuda:0")
