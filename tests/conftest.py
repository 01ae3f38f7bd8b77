import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: full-size configuration (minutes)")


def _has_cuda():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


def pytest_collection_modifyitems(config, items):
    if _has_cuda():
        return
    skip = pytest.mark.skip(reason="no CUDA device")
    for it in items:
        if "gpu" in it.keywords:
            it.add_marker(skip)


_PARITY = {}


@pytest.fixture(scope="session")
def parity_report():
    """name -> (worst err/limit, elements compared) of the full-size parity tests (printed at the end)."""
    return _PARITY


def pytest_terminal_summary(terminalreporter, exitstatus, config):
    if not _PARITY:
        return
    terminalreporter.write_sep("-", "full-size parity vs oracle O1 (every element compared)")
    for k, (worst, n) in sorted(_PARITY.items()):
        terminalreporter.write_line(f"{k:32s} {n:>13,d} elements  worst err/limit {worst:.4f}")
