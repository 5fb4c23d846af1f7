import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

GOLDEN = os.path.join(ROOT, "tests", "golden")


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (sm_100a) GPU; parity tests through the C-ABI")
    config.addinivalue_line("markers", "slow: long-running")


def read_golden(name):
    rows = []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                rows.append(line.split())
    return rows


def golden_facts(name):
    """'# key value' lines after the table."""
    facts = {}
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            parts = line.strip().lstrip("#").split()
            if len(parts) == 2:
                try:
                    facts[parts[0]] = float(parts[1])
                except ValueError:
                    pass
    return facts


@pytest.fixture(scope="session")
def orc():
    import oracle
    oracle.lib()
    return oracle
