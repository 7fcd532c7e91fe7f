#!/bin/bash
# round-2 full check: all gpu tests, smoke, default bench (MoE headline + GPT also), GPT tc-attention A/B
O=gpurun_out
mkdir -p $O
rm -f $O/parity_log.jsonl
timeout 1500 python -m pytest tests -m gpu -q -rf --timeout 300 > $O/pt_full.txt 2>&1; echo "pytest rc=$?" >> $O/pt_full.txt
timeout 300 python __graft_entry__.py smoke > $O/smoke.txt 2>&1; echo "smoke rc=$?" >> $O/smoke.txt
timeout 900 python bench.py > $O/bench.json 2>$O/bench.err; echo "bench rc=$?" >> $O/bench.err
PREDTOP_ATTN_TC=1 timeout 300 python bench.py --config gpt --no-cpu-baseline --no-also --steps 20 > $O/bench_gpt_tc.json 2>$O/bench_gpt_tc.err
tail -6 $O/pt_full.txt; tail -2 $O/smoke.txt; tail -2 $O/bench.err
python - <<'PY'
import json
for f in ["gpurun_out/bench.json", "gpurun_out/bench_gpt_tc.json"]:
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f, d["value"], d["unit"], "ms/step", round(d["ms_per_step"], 4), "parity", d.get("parity"))
        print({k: round(v["ms_per_step"], 3) for k, v in d.get("kernels", {}).items()})
        g = d.get("also", {}).get("gpt")
        if g: print("gpt", g["value"], g["ms_per_step"], g.get("parity"))
    except Exception as e:
        print(f, "parse failed", e)
PY
