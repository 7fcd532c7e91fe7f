import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA sm_100 device (B200)")
    config.addinivalue_line("markers", "slow: long-running CPU test")


@pytest.fixture(scope="session")
def oracle_mod():
    import oracle
    oracle.build()
    return oracle


@pytest.fixture(scope="session")
def parity_log():
    """record(name, **fields): append one JSON line of measured GPU-vs-oracle
    errors to $PREDTOP_PARITY_LOG (default gpurun_out/parity_log.jsonl, which
    gpurun brings back; profiles/parity_r02.json is the tracked copy)."""
    import json
    import time
    path = os.environ.get("PREDTOP_PARITY_LOG", os.path.join(ROOT, "gpurun_out", "parity_log.jsonl"))

    def record(name, **fields):
        try:
            os.makedirs(os.path.dirname(path), exist_ok=True)
            with open(path, "a") as f:
                f.write(json.dumps(dict(test=name, when=time.strftime("%Y-%m-%dT%H:%M:%S"),
                                        **{k: (float(v) if hasattr(v, "dtype") else v)
                                           for k, v in fields.items()})) + "\n")
        except OSError:
            pass
    return record

