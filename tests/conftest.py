import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA GPU (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running test")


@pytest.fixture(scope="session")
def cuda_available():
    import torch
    return torch.cuda.is_available()


@pytest.fixture
def tune():
    """Set libhmg performance knobs (hmg_set_tuning) for one test; all cleared afterwards."""
    from paper_conf_ipps_jiangg15_b200 import hmg
    hmg.lib()

    def set_(name, value):
        hmg.set_tuning(name, int(value))
    yield set_
    hmg.clear_tuning()
