import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200); run with -m gpu")
    config.addinivalue_line("markers", "slow: long-running test")


@pytest.fixture(scope="session")
def oracle_mod():
    import oracle
    oracle.build()
    return oracle


def pytest_sessionfinish(session, exitstatus):
    """Totals of the parity comparisons of this session (band_only_* counts:
    pairs excused by the tie band) -> gpurun_out/parity_summary.json."""
    try:
        import dts_parity
    except ImportError:
        return
    if not dts_parity.SUMMARY:
        return
    import json
    out = os.path.join(ROOT, "gpurun_out")
    os.makedirs(out, exist_ok=True)
    tot = {k: sum(s[k] for s in dts_parity.SUMMARY)
           for k in ("gpu", "oracle", "common", "band_only_gpu", "band_only_oracle")}
    tot["comparisons"] = len(dts_parity.SUMMARY)
    tot["worst_endpoint"] = max(s["worst_endpoint"] for s in dts_parity.SUMMARY)
    tot["excused"] = [s for s in dts_parity.SUMMARY if s["band_only_gpu"] or s["band_only_oracle"]]
    with open(os.path.join(out, "parity_summary.json"), "w") as f:
        json.dump(tot, f, indent=1)
