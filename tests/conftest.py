import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (sm_100a) GPU; run with -m gpu")
    config.addinivalue_line("markers", "slow: long-running CPU test")


@pytest.fixture(scope="session")
def lib():
    """The C-ABI library through the thin ctypes binding (builds it if missing)."""
    from paper_conf_asplos_xiazswwyfc24_b200 import _lib
    return _lib.load()


@pytest.fixture
def record_err(request):
    """Append a parity test's achieved error next to its tolerance to a JSONL log (default
    gpurun_out/parity_errors.jsonl, or $SOUFFLE_ERR_LOG), so the margin under each tolerance is kept."""
    import json

    def rec(err, tol, **extra):
        path = os.environ.get("SOUFFLE_ERR_LOG", os.path.join(ROOT, "gpurun_out", "parity_errors.jsonl"))
        os.makedirs(os.path.dirname(path), exist_ok=True)
        with open(path, "a") as f:
            f.write(json.dumps(dict(test=request.node.nodeid, err=float(err), tol=float(tol), **extra)) + "\n")
        assert err <= tol, (request.node.nodeid, err, tol, extra)
    return rec
