#!/bin/bash
# GPU-box helper: the full round-end set (tests, smoke, every bench config,
# reference arm, ncu launch list).  Outputs land in gpurun_out/.
set -x
O=gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $O/pt.txt 2>&1
timeout 300 python __graft_entry__.py smoke > $O/smoke.txt 2>&1
timeout 400 python bench.py > $O/bench_gpt.json 2>$O/bench_gpt.err
for c in tiny moe 16k sweep; do
  timeout 400 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline > $O/bench_$c.json 2>$O/bench_$c.err
done
timeout 400 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_ref.json 2>$O/bench_ref.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches.csv python tools/prof_step.py --warmup 1 --steps 1 > $O/ncu_ll.log 2>&1
timeout 400 python bench.py --config search --steps 10 --warmup 3 --no-cpu-baseline > $O/bench_search.json 2>$O/bench_search.err
timeout 300 python bench.py --hops 4 --steps 30 --warmup 5 --no-cpu-baseline > $O/bench_hops4.json 2>$O/bench_hops4.err
