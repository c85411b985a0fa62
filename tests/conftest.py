import json
import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

GOLDEN = os.path.join(ROOT, "tests", "golden")


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (CUDA) -- parity tests through the C-ABI")
    config.addinivalue_line("markers", "slow: long-running (large sizes)")


def load_golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


@pytest.fixture(scope="session")
def e1():
    return load_golden("e1.json")


@pytest.fixture(scope="session")
def e2():
    return load_golden("e2.json")


@pytest.fixture(scope="session")
def paper_arith():
    return load_golden("paper_arith.json")


@pytest.fixture(scope="session")
def golden():
    return lambda name: load_golden(name + ".json")
