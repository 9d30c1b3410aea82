import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running (full-size oracle runs)")


def cuda_available() -> bool:
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


@pytest.fixture(scope="session")
def need_gpu():
    if not cuda_available():
        pytest.fail("CUDA device required for -m gpu tests (no silent skip: the GPU tier must run on a GPU box)")


def pytest_sessionfinish(session, exitstatus):
    path = os.environ.get("BTED_PARITY_REPORT")
    if not path:
        return
    import json
    try:
        from tests.parity import REPORT
    except Exception:
        return
    if REPORT:
        os.makedirs(os.path.dirname(os.path.abspath(path)), exist_ok=True)
        worst = max(r["max_rel_score_err"] for r in REPORT)
        with open(path, "w") as f:
            json.dump({"calls": len(REPORT), "worst_max_rel_score_err": worst,
                       "total_steps": sum(r["steps"] for r in REPORT),
                       "total_near_ties": sum(r["near_ties"] for r in REPORT), "runs": REPORT}, f, indent=1)
