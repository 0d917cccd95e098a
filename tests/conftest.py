import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    # A fresh checkout has no libeatss.so (built artefacts are not tracked): build it
    # (and the C oracle) once, the same way __graft_entry__.build() does.
    if not os.path.exists(os.path.join(ROOT, "paper_conf_cgo_jayaweerakwk24_b200", "libeatss.so")):
        import __graft_entry__

        __graft_entry__.build()
    config.addinivalue_line("markers", "gpu: needs a CUDA B200 (sm_100a) device")
    config.addinivalue_line("markers", "slow: long-running CPU test")


@pytest.fixture(scope="session")
def cuda_device():
    import torch

    if not torch.cuda.is_available():
        pytest.fail("gpu test selected but no CUDA device is visible")
    return torch.device("cuda:0")
