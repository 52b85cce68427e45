import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running CPU test")


def _ensure_oracle_built():
    src = os.path.join(ROOT, "oracle", "snn_oracle.c")
    lib = os.path.join(ROOT, "oracle", "liboracle.so")
    if (not os.path.exists(lib)) or os.path.getmtime(lib) < os.path.getmtime(src):
        import __graft_entry__  # noqa: E402
        __graft_entry__.build_oracle()


def _ensure_cuda_built():
    lib = os.path.join(ROOT, "paper_conf_date_shelm19_b200", "libsnn_b200.so")
    csrc = os.path.join(ROOT, "paper_conf_date_shelm19_b200", "csrc")
    newest = max(os.path.getmtime(os.path.join(csrc, f)) for f in os.listdir(csrc))
    newest = max(newest, os.path.getmtime(os.path.join(ROOT, "include", "snn.h")))
    if (not os.path.exists(lib)) or os.path.getmtime(lib) < newest:
        import __graft_entry__  # noqa: E402
        __graft_entry__.build_cuda()


_ensure_oracle_built()
_ensure_cuda_built()


def cuda_available() -> bool:
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


@pytest.fixture(scope="session")
def gpu():
    if not cuda_available():
        pytest.skip("no CUDA device")
    return True
