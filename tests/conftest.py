import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); run with -m gpu")
    config.addinivalue_line("markers", "slow: long-running (minutes); excluded unless selected")


def pytest_collection_modifyitems(config, items):
    # `slow` tests only run when explicitly selected with -m containing "slow".
    markexpr = config.getoption("-m") or ""
    if "slow" in markexpr:
        return
    skip = pytest.mark.skip(reason="slow test: select with -m slow")
    for it in items:
        if "slow" in it.keywords:
            it.add_marker(skip)


def _ensure_lib():
    """Build libhdb.so in-tree if missing (nvcc cross-compiles without a GPU)."""
    import paper_conf_ipps_gowanlockrblp17_b200 as pkg
    if not os.path.exists(pkg.LIB_PATH):
        pkg.build()


_ensure_lib()


def cuda_available():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False
