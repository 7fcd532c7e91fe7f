"""The multi-rank product path through bench.py (north star:
graphs sharded over ranks, ONE all-gather of the fp64 plan latencies, the
same global argmin on every rank).  Two ranks share the one GPU of the test
box through the gloo backend (NCCL refuses two ranks on one device); each
rank builds and scores its own GPU shard, so the gathered T is made by the
GPU path, and it must be bitwise the 1-rank result over the union of the
shards (weak scaling: rank r owns graphs [G r, G (r+1)))."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
pytestmark = pytest.mark.gpu


def _bench(*args):
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--config", "gpt", "--steps", "3",
                        "--warmup", "3", "--no-extras"] + list(args),
                       capture_output=True, text=True, timeout=900, cwd=ROOT,
                       env={k: v for k, v in os.environ.items() if k not in ("RANK", "WORLD_SIZE", "LOCAL_RANK")})
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-3000:]
    return json.loads(lines[0])


def test_two_ranks_gather_bitwise_equal_to_one_rank():
    one = _bench("--graphs", "64", "--eager")
    two = _bench("--graphs", "32", "--gpus", "2", "--dist-backend", "gloo")
    assert one["n_gpus"] == 1 and two["n_gpus"] == 2
    assert one["result"]["plans"] == two["result"]["plans"] == 16
    assert two["result"]["T_sha256"] == one["result"]["T_sha256"]
    assert two["result"]["best_plan"] == one["result"]["best_plan"]
    assert two["value"] > 0
