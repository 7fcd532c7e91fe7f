#!/bin/bash
# round-2 final evidence (last session): full gpu tests, smoke, default bench (MoE headline + GPT also),
# the other configs, training bench, ncu launch list of the MoE bench
O=gpurun_out; mkdir -p $O
rm -f $O/parity_log.jsonl
timeout 1500 python -m pytest tests -m gpu -q -rf --timeout 300 > $O/pt_full.txt 2>&1; echo "pytest rc=$?" >> $O/pt_full.txt
timeout 300 python __graft_entry__.py smoke > $O/smoke.txt 2>&1; echo "smoke rc=$?" >> $O/smoke.txt
timeout 900 python bench.py > $O/bench.json 2>$O/bench.err; echo "bench rc=$?" >> $O/bench.err
tail -3 $O/pt_full.txt; tail -2 $O/smoke.txt; tail -1 $O/bench.err
for c in 16k search sweep tiny; do
  timeout 900 python bench.py --config $c > $O/bench_cfg_$c.json 2>$O/bench_cfg_$c.err; echo "$c rc=$?"
done
timeout 600 python bench.py --config train --no-cpu-baseline > $O/bench_train.json 2>$O/bench_train.err; echo "train rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_moe.csv python bench.py --config moe --no-cpu-baseline --no-also --steps 2 --warmup 1 > $O/ncu_launch.log 2>&1; echo "ncu rc=$?"
python - <<'PY'
import json
for f in ["bench.json", "bench_cfg_16k.json", "bench_cfg_search.json", "bench_cfg_sweep.json", "bench_cfg_tiny.json", "bench_train.json"]:
    try:
        d = json.loads(open("gpurun_out/" + f).read().strip().splitlines()[-1])
        print(f, round(d["value"], 1), d["unit"], "ms/step", round(d["ms_per_step"], 4), "frac", (d.get("roofline") or {}).get("frac"), "parity", (d.get("parity") or {}).get("max_rel"))
        g = d.get("also", {}).get("gpt")
        if g: print("  gpt", g["value"], g["ms_per_step"], (g.get("parity") or {}).get("max_rel"))
    except Exception as e:
        print(f, "parse failed", e)
PY
