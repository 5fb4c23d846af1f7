import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

GOLDEN = os.path.join(ROOT, "tests", "golden")


if os.environ.get("PAGODA_TEST_FLAGS"):
    # run the suite with extra context flags (e.g. PAGODA_TEST_FLAGS=0x40: every context uses the
    # copy-engine ingest): pagoda_config.flags of every context the tests create is OR-ed with them
    from paper_conf_ppopp_yehsser17_b200 import pagoda as _pg
    _extra = int(os.environ["PAGODA_TEST_FLAGS"], 0)
    _default_config = _pg.default_config

    def _with_flags(**kw):
        cfg = _default_config(**kw)
        cfg.flags |= _extra
        return cfg
    _pg.default_config = _with_flags


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
