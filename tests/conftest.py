import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (runs the CUDA path through the C ABI)")
    config.addinivalue_line("markers", "slow: full-size parity runs")


def _make(target):
    subprocess.run(["make", "-C", ROOT, target], check=True, stdout=subprocess.DEVNULL)


@pytest.fixture(scope="session", autouse=True)
def _host_libs():
    """Build the gcc-only libraries (oracle, synth) if they are missing."""
    if not (os.path.exists(os.path.join(ROOT, "oracle", "liboracle.so"))
            and os.path.exists(os.path.join(ROOT, "synth", "libsynth.so"))):
        _make("host")
    yield


def gpu_available():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


@pytest.fixture(scope="session")
def ap():
    """The product binding (loads libapointer.so; fails loudly if missing)."""
    lib = os.path.join(ROOT, "paper_conf_isca_shaharbs16_b200", "libapointer.so")
    if not os.path.exists(lib):
        _make("all")
    import paper_conf_isca_shaharbs16_b200 as ap_mod
    return ap_mod
