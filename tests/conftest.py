import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running CPU test")


def gpu_available():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


def pytest_collection_modifyitems(config, items):
    if gpu_available():
        return
    skip = pytest.mark.skip(reason="no CUDA device")
    for it in items:
        if "gpu" in it.keywords:
            it.add_marker(skip)


@pytest.fixture
def options():
    """set_option(name, value) that restores every touched option afterwards."""
    import paper_conf_sc_augonnetasg24_b200 as stf

    saved = {}

    def setter(name, value):
        if name not in saved:
            saved[name] = stf.get_option(name)
        stf.set_option(name, value)

    yield setter
    for k, v in saved.items():
        stf.set_option(k, v)
