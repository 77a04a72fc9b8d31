import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running CPU test")


def pytest_collection_modifyitems(config, items):
    try:
        import torch
        has_gpu = torch.cuda.is_available()
    except Exception:  # pragma: no cover
        has_gpu = False
    if has_gpu:
        return
    skip = pytest.mark.skip(reason="no CUDA device")
    for it in items:
        if "gpu" in it.keywords:
            it.add_marker(skip)


@pytest.fixture(autouse=True)
def _reset_spinfer_options():
    """Library options (kernel choice, grid cap, stage shape) are process-wide: every test
    starts and ends with the defaults."""
    yield
    mod = sys.modules.get("paper_conf_eurosys_fanydlgww025_b200")
    if mod is not None and getattr(mod, "_lib", None) is not None:
        for name in mod.OPTIONS:
            mod.set_option(name, 0)
