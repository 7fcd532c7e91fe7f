#!/bin/bash
# GPU-box helper (round 2): gpu tests (all, no -x), smoke, default bench
# (MoE headline + GPT under "also").  Outputs land in gpurun_out/.
O=gpurun_out
mkdir -p $O
rm -f $O/parity_log.jsonl
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt 2>&1
timeout ${PT_TIMEOUT:-1500} python -m pytest tests -m gpu -q -rf --durations=20 ${PT_ARGS} > $O/pt.txt 2>&1; echo "pytest rc=$?" >> $O/pt.txt
timeout 300 python __graft_entry__.py smoke > $O/smoke.txt 2>&1; echo "smoke rc=$?" >> $O/smoke.txt
timeout 900 python bench.py ${BENCH_ARGS} > $O/bench.json 2>$O/bench.err; echo "bench rc=$?" >> $O/bench.err
tail -15 $O/pt.txt; tail -2 $O/smoke.txt; tail -3 $O/bench.err
python - <<'PY'
import json
try:
    d = json.loads(open("gpurun_out/bench.json").read().strip().splitlines()[-1])
    print(d["value"], d["unit"], "ms/step", round(d["ms_per_step"], 4), "parity", d.get("parity"))
    print({k: round(v["ms_per_step"], 3) for k, v in d.get("kernels", {}).items()})
    g = d.get("also", {}).get("gpt")
    if g: print("gpt", g["value"], g["ms_per_step"], g.get("parity"))
except Exception as e:
    print("bench parse failed", e)
PY
