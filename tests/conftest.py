import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running")


def has_gpu():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


@pytest.fixture(scope="session")
def gpu():
    if not has_gpu():
        pytest.skip("no CUDA device")
    import torch
    return torch.device("cuda:0")


def expected_selection(rep, ids, default_vid):
    """The device selection rule on a report (oracle.selection.select_with_margin,
    DESIGN.md A-50) over the pool's variant ids: argmin of the scores (ties ->
    pool order) unless the initial version's completed score is within 1/9."""
    from oracle import selection
    scores = [rep["score"][v] for v in ids]
    return ids[selection.select_with_margin(scores, ids.index(default_vid))]
