#!/bin/bash
# GPU-box helper: attention-focused parity tests + MoE/GPT bench lines.
O=gpurun_out
mkdir -p $O
rm -f $O/parity_log.jsonl
timeout ${PT_TIMEOUT:-600} python -m pytest tests -m gpu -q -x -rf ${PT_ARGS:--k "moe or tc or tiny"} > $O/pt_attn.txt 2>&1; echo "pytest rc=$?" >> $O/pt_attn.txt
tail -5 $O/pt_attn.txt
for cfg in ${BENCH_CFGS:-moe}; do
  timeout 600 python bench.py --config $cfg --no-cpu-baseline ${BENCH_ARGS} > $O/bench_$cfg.json 2>$O/bench_$cfg.err; echo "bench $cfg rc=$?"
  python - $cfg <<'PY'
import json, sys
cfg = sys.argv[1]
try:
    d = json.loads(open(f"gpurun_out/bench_{cfg}.json").read().strip().splitlines()[-1])
    print(cfg, d["value"], d["unit"], "ms/step", round(d["ms_per_step"], 4))
    print({k: round(v["ms_per_step"], 3) for k, v in d.get("kernels", {}).items()})
    print("roofline", d.get("roofline"))
except Exception as e:
    print("bench parse failed", e); print(open(f"gpurun_out/bench_{cfg}.err").read()[-2000:])
PY
done
