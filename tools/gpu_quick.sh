#!/bin/bash
# GPU-box helper for iterations: gpu tests + a short GPT bench (+ optional
# extra bench args as "$@").  Outputs land in gpurun_out/.
O=gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q > $O/pt.txt 2>&1; echo "pytest rc=$?" >> $O/pt.txt
timeout 300 python bench.py --steps 30 --warmup 5 --no-cpu-baseline "$@" > $O/bench_q.json 2>$O/bench_q.err
tail -3 $O/pt.txt
python - <<'PY'
import json
d = json.loads(open("gpurun_out/bench_q.json").read().strip().splitlines()[-1])
print(d["value"], d["unit"], "ms/step", round(d["ms_per_step"], 4))
print({k: round(v["ms_per_step"], 3) for k, v in d.get("kernels", {}).items()})
PY
