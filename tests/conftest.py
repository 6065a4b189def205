import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (sm_100a) GPU; run via gpurun")
    config.addinivalue_line("markers", "slow: long-running CPU test")


@pytest.fixture(scope="session")
def golden():
    import json
    with open(os.path.join(ROOT, "tests", "golden", "paper_examples.json")) as f:
        return json.load(f)


def pytest_sessionfinish(session, exitstatus):
    mod = sys.modules.get("gpu_helpers")
    rec = getattr(mod, "RECORD", None) if mod else None
    if rec:
        import json
        out = os.environ.get("VB_PARITY_OUT", os.path.join(ROOT, "gpurun_out", "parity.json"))
        os.makedirs(os.path.dirname(out), exist_ok=True)
        with open(out, "w") as f:
            json.dump({"exitstatus": int(exitstatus), "cases": rec}, f, indent=1, sort_keys=True)
