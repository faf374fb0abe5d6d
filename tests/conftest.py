import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (sm_100a) GPU; run with -m gpu")
    config.addinivalue_line("markers", "slow: long-running test")


@pytest.fixture(scope="session")
def cuda_device():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("GPU test selected but no CUDA device is visible")
    return torch.device("cuda:0")


def pytest_sessionfinish(session, exitstatus):
    """Dump the achieved parity errors the GPU tests recorded (tests/parity_log.py)."""
    try:
        from tests import parity_log
    except ImportError:
        try:
            import parity_log
        except ImportError:
            return
    if not parity_log.RECORDS:
        return
    import json
    out = os.path.join(ROOT, "gpurun_out")
    os.makedirs(out, exist_ok=True)
    with open(os.path.join(out, "parity_errors.jsonl"), "w") as f:
        for r in parity_log.RECORDS:
            f.write(json.dumps(r) + "\n")
