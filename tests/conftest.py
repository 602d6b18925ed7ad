import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA GPU (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: longer-running CPU test")


def _has_gpu():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


def pytest_collection_modifyitems(config, items):
    if _has_gpu():
        return
    skip = pytest.mark.skip(reason="no CUDA GPU in this container")
    for it in items:
        if "gpu" in it.keywords:
            it.add_marker(skip)


@pytest.fixture(scope="session")
def ctx():
    """Single-process, single-GPU context (the bench's N=1 configuration)."""
    import torch

    from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

    torch.cuda.set_device(0)
    c = M.mapsm_ctx_create(0, 1, 0, None, None)
    yield c
    M.mapsm_ctx_destroy(c)


@pytest.fixture(scope="session")
def local_ctx():
    """Factory: single-process g-slab context on cuda:0 (halo exchange by D2D copies)."""
    from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

    made = {}

    def make(g):
        if g not in made:
            made[g] = M.mapsm_ctx_create_local([0] * g)
        return made[g]

    yield make
    for c in made.values():
        M.mapsm_ctx_destroy(c)
