import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")


def have_gpu() -> bool:
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


@pytest.fixture(scope="session")
def oracle_mod():
    import oracle
    oracle.build()
    return oracle


# Device selection from online profiles redirects repeated COOP launches of a
# shape to one device; the parity tests exercise the cooperative path itself, so contexts
# created by the tests default to it off (tests/test_gpu_select.py turns it on per launch).
os.environ.setdefault("FCL_SELECT", "0")
