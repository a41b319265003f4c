import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def _ensure_built():
    """Build the CUDA library (nvcc cross-compiles without a GPU) and the C
    oracle if they are missing, so a fresh checkout can run the CPU suite."""
    lib = os.path.join(ROOT, "paper_conf_cgo_gonzalohghmh19_b200", "libreduce_b200.so")
    if not os.path.exists(lib):
        import importlib.util  # load _build.py alone: the package itself needs the .so
        spec = importlib.util.spec_from_file_location(
            "_rb_build", os.path.join(ROOT, "paper_conf_cgo_gonzalohghmh19_b200", "_build.py"))
        mod = importlib.util.module_from_spec(spec)
        spec.loader.exec_module(mod)
        mod.build()


_ensure_built()


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA B200 (run with -m gpu on the GPU box)")
    config.addinivalue_line("markers", "slow: long-running (full-size parity)")


def _has_cuda():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


def pytest_collection_modifyitems(config, items):
    if _has_cuda():
        return
    skip = pytest.mark.skip(reason="no CUDA device in this container")
    for item in items:
        if "gpu" in item.keywords:
            item.add_marker(skip)
