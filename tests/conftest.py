import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running CPU test")
    # Build the native artefacts this checkout lacks (they are git-ignored).
    import __graft_entry__ as ge
    if not os.path.exists(os.path.join(ROOT, "oracle", "liboracle.so")):
        ge.build_oracle()
    if not os.path.exists(os.path.join(ROOT, "gen", "libmagus_gen.so")):
        ge.build_gen()
    if (os.path.isdir(os.path.join(ROOT, "paper_conf_sc_zhengspl25_b200"))
            and not os.path.exists(os.path.join(ROOT, "paper_conf_sc_zhengspl25_b200", "libmagus.so"))):
        from paper_conf_sc_zhengspl25_b200 import _build
        _build.build_libmagus()


def _cuda_ok() -> bool:
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


def pytest_collection_modifyitems(config, items):
    if _cuda_ok():
        return
    skip = pytest.mark.skip(reason="no CUDA device")
    for it in items:
        if "gpu" in it.keywords:
            it.add_marker(skip)
