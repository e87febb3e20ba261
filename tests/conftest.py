import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); parity tests through the C-ABI")
    config.addinivalue_line("markers", "slow: long-running CPU test")


@pytest.fixture(scope="session")
def oracle_mod():
    import oracle
    oracle.build()
    return oracle


def pytest_terminal_summary(terminalreporter):
    """Every parity comparison's taint counts (reading C13) in the log: tainted
    pairs are compared and reported, never silently excluded."""
    try:
        from tests.parity import REPORT
    except Exception:
        return
    if not REPORT:
        return
    terminalreporter.write_sep("-", "parity taint report (F mode: tainted pairs compared, not asserted)")
    for label, r in REPORT:
        terminalreporter.write_line(
            f"{label}: pairs={r['pairs']} tainted={r['tainted']} ({100 * r['tainted_frac']:.2f}%) "
            f"tainted_differ={r['tainted_differ']} flags={r['flags']} events={r['events']} "
            f"max_err={r['max_time_err']:.3g}")
