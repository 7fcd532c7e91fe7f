"""bench.py's non-default configs end to end on the GPU (small sizes): the
driver only runs the default (MoE) line, so a config-specific code path
(e.g. the sweep's oracle cpu_baseline) could otherwise break unseen.  Each
line must carry the contract keys."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
pytestmark = pytest.mark.gpu

CONTRACT = ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
            "dtype", "data", "config", "e2e", "gpu_launches", "clocks")


def _bench(*args):
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + list(args),
                       capture_output=True, text=True, timeout=900, cwd=ROOT,
                       env={k: v for k, v in os.environ.items() if k not in ("RANK", "WORLD_SIZE", "LOCAL_RANK")})
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-3000:]
    return json.loads(lines[0])


def test_sweep_line_with_cpu_baseline():
    d = _bench("--config", "sweep", "--plans", "2000", "--pool", "512", "--chunk", "256", "--steps", "1",
               "--warmup", "3")
    for k in CONTRACT:
        assert k in d, k
    assert d["value"] > 0 and d["e2e"]["value"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["value"] > 0
    assert d["roofline"]["frac"] > 0


def test_tiny_line():
    d = _bench("--config", "tiny", "--steps", "5", "--warmup", "3")
    for k in CONTRACT:
        assert k in d, k
    assert d["value"] > 0 and d["gpu_launches"] > 0
    assert d["parity"]["pass"]
