import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (sm_100a) GPU")
    config.addinivalue_line("markers", "slow: long-running (still CPU-only unless also marked gpu)")


_built = False


def _build(targets):
    subprocess.run(["make", "-s", "-C", ROOT, "-j8"] + targets, check=True)


@pytest.fixture(scope="session", autouse=True)
def native_libs():
    """Build the in-tree native libraries once per session (make is incremental)."""
    global _built
    if not _built:
        targets = ["gen/libvista_gen.so", "oracle/liboracle.so"]
        if os.path.exists("/usr/local/cuda/bin/nvcc") and os.path.exists(os.path.join(ROOT, "paper_conf_sigmod_nakandalak20_b200/csrc/vista_api.cpp")):
            targets.append("paper_conf_sigmod_nakandalak20_b200/libvista.so")
        _build(targets)
        _built = True
    yield


def has_gpu():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False
