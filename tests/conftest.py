import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA GPU (B200); run with -m gpu")
    config.addinivalue_line("markers", "slow: long CPU test")


def _ensure_built():
    libs = ["lt_inputs/libltgen.so", "oracle/liboracle.so", "paper_conf_icde_xing0wxl23_b200/liblt.so"]
    if not all(os.path.exists(os.path.join(ROOT, p)) for p in libs):
        subprocess.run(["make", "-C", ROOT, "-j8", "all"], check=False, capture_output=True)


_ensure_built()


def has_gpu():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


@pytest.fixture(scope="session")
def gpu():
    if not has_gpu():
        pytest.fail("test marked gpu but no CUDA device is visible")
    return 0
