#!/bin/bash
# round-2 final evidence: full gpu tests, smoke, default bench (MoE headline + GPT),
# training bench, ncu launch list of the MoE bench, compute-sanitizer
O=gpurun_out; mkdir -p $O
bash tools/gpu_full2.sh
timeout 600 python bench.py --config train --no-cpu-baseline > $O/bench_train.json 2>$O/bench_train.err; tail -c 400 $O/bench_train.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_moe.csv python bench.py --config moe --no-cpu-baseline --no-also --steps 2 --warmup 1 > $O/ncu_launch.log 2>&1; echo "ncu rc=$?"
bash tools/gpu_sanitize.sh
