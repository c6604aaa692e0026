import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); run on the GPU box")
    config.addinivalue_line("markers", "slow: takes more than ~10 s")


@pytest.fixture(scope="session")
def golden_expected():
    import json
    with open(os.path.join(ROOT, "tests", "golden", "expected.json")) as f:
        return json.load(f)
