import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (run via gpurun)")
    config.addinivalue_line("markers", "host: CPU-only host logic")
    config.addinivalue_line("markers", "slow: long-running CPU test")
    config.addinivalue_line("markers", "multigpu: needs >= 2 GPUs; runs only with -m multigpu")


def pytest_collection_modifyitems(config, items):
    # multi-GPU tests run only when explicitly selected (-m multigpu): the driver's
    # 1-GPU "-m gpu" tier and the CPU tier never see them
    if "multigpu" in (config.option.markexpr or ""):
        return
    keep = [it for it in items if it.get_closest_marker("multigpu") is None]
    if len(keep) != len(items):
        config.hook.pytest_deselected(items=[it for it in items if it not in keep])
        items[:] = keep


@pytest.fixture(scope="session")
def cuda_device():
    import torch
    if not torch.cuda.is_available():
        # gpu tests run only where a GPU is promised: a silent skip would read as a pass
        pytest.fail("gpu-marked test but torch.cuda.is_available() is False")
    return torch.device("cuda:0")
