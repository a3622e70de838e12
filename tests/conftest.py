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
    """The device selection rule on a report: the argmin of the live scores
    (ties -> pool order), except that a challenger must predict more than
    1/9 faster than the initial version's own completed score (switch margin,
    DESIGN.md A-50)."""
    cap = (1 << 56) - 1
    live = [v for v in ids if rep["score"][v] != cap]
    best = min(live, key=lambda v: (rep["score"][v], ids.index(v)))
    if best != default_vid and default_vid in live and rep["score"][best] * 9 > rep["score"][default_vid] * 8:
        return default_vid
    return best
