import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a) and libtbs.so")
    config.addinivalue_line("markers", "slow: long CPU test (oracle at large n)")


@pytest.fixture(scope="session")
def tbs():
    """The product binding (GPU tests only)."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import paper_conf_icpp_pitaksirianannt16_b200 as t
    return t
