import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); run with -m gpu")
    config.addinivalue_line("markers", "slow: long-running CPU test")


def gpu_status():
    try:
        import torch
        ok = torch.cuda.is_available()
        return ok, f"torch {torch.__version__} cuda.is_available()={ok} count={torch.cuda.device_count()} " \
                   f"CUDA_VISIBLE_DEVICES={os.environ.get('CUDA_VISIBLE_DEVICES')}"
    except Exception as e:  # report the real reason
        return False, f"{type(e).__name__}: {e}"


@pytest.fixture(scope="session")
def gpu():
    ok, why = gpu_status()
    if not ok:
        pytest.fail(f"GPU test without a usable CUDA device: {why}")
    return 0
