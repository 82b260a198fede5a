import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA (sm_100) device")
    config.addinivalue_line("markers", "slow: long-running (large graph) case")


def pytest_collection_modifyitems(config, items):
    try:
        import torch

        has_gpu = torch.cuda.is_available()
    except Exception:  # pragma: no cover
        has_gpu = False
    if has_gpu:
        return
    skip = pytest.mark.skip(reason="no CUDA device")
    for item in items:
        if "gpu" in item.keywords:
            item.add_marker(skip)


@pytest.fixture(autouse=True)
def _release_library_cache():
    """Every test leaves the GPU as it found it: the library's cached device
    blocks go back to the driver (PyTorch allocates the next test's graph)."""
    yield
    try:
        import gc

        import torch

        if not torch.cuda.is_available():
            return
        import paper_conf_ipps_geilpo23_b200 as m

        gc.collect()  # graph handles a test did not close free their workspaces first
        m.empty_cache(torch.cuda.current_device())
    except Exception:  # pragma: no cover  (no library built: nothing cached)
        pass
