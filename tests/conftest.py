import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); parity tests of the CUDA path")
    config.addinivalue_line("markers", "slow: long-running")
    # Build native artefacts if missing or stale (cheap no-op when up to date).
    targets = ["ragen/libragen.so", "oracle/liboracle.so"]
    if os.path.exists(os.path.join(ROOT, "include", "ra.h")):
        targets.append("paper_conf_ipps_wudwcyc12_b200/libra.so")
    r = subprocess.run(["make", "-s", "-C", ROOT, *targets], capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("native build failed:\n" + r.stdout + r.stderr)


def pytest_collection_modifyitems(config, items):
    try:
        import torch
        has_gpu = torch.cuda.is_available()
    except Exception:  # pragma: no cover
        has_gpu = False
    if has_gpu:
        return
    skip = pytest.mark.skip(reason="no CUDA device in this container (run with -m gpu on a B200)")
    for item in items:
        if "gpu" in item.keywords:
            item.add_marker(skip)


@pytest.fixture(autouse=True)
def _release_device_memory():
    """Several parity tests hold tens of GB on the device (full-size configs,
    row-limit tests); return cached blocks after each test so later ones start
    from an empty pool."""
    yield
    try:
        import torch
        if torch.cuda.is_available():
            import gc
            gc.collect()
            torch.cuda.empty_cache()
    except Exception:  # pragma: no cover
        pass
