import os
import sys
from pathlib import Path

import pytest

ROOT = Path(__file__).resolve().parent.parent
if str(ROOT) not in sys.path:
    sys.path.insert(0, str(ROOT))


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: longer CPU test")


@pytest.fixture(scope="session")
def orc():
    import oracle
    oracle.lib()
    return oracle


def pytest_terminal_summary(terminalreporter):
    """Totals of the parity comparisons run this session: rows matched element by element and
    rows set aside by the parity rules' exclusions (threshold/owner-boundary/MULTI), per kind."""
    par = sys.modules.get("tests.parity") or sys.modules.get("parity")
    if par is None or not getattr(par, "TALLY", None):
        return
    tot = {}
    for kind, m, e in par.TALLY:
        a = tot.setdefault(kind, [0, 0, 0])
        a[0] += 1
        a[1] += m
        a[2] += e
    terminalreporter.write_line("parity exclusions: " + "; ".join(
        f"{k}: {c} comparisons, {m} matched, {e} excluded ({e / max(1, m + e):.2e})"
        for k, (c, m, e) in sorted(tot.items())))
    for (test, why), c in sorted(getattr(par, "REASONS", {}).items()):
        terminalreporter.write_line(f"  excluded conjunctions, {why}: {c}  ({test})")
