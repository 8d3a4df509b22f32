import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
# Virtual ranks (several handles on one GPU, tests/test_gpu_join.py) wait for
# each other inside kernels on up to two streams per rank: every stream needs
# its own hardware queue, or a waiting kernel can hold back a peer's work
# queued behind it (CUDA's default is 8 queues).  Must be set before CUDA starts.
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA B200 (run on the GPU box)")
    config.addinivalue_line("markers", "slow: full-size configurations")


@pytest.fixture(scope="session")
def cuda_available():
    import torch
    return torch.cuda.is_available()
