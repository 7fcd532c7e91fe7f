#!/bin/bash
# GPU-box helper: parity + bench of the main build and debug/variant builds
# lib/libpredtop_<v>.so given as arguments.  Outputs land in gpurun_out/.
L=$PWD/paper_conf_ipps_acharyas25_b200/lib
timeout 120 python tools/repeat_check.py > gpurun_out/rc.txt 2>&1
for v in "$@"; do echo "== $v" >> gpurun_out/rc.txt; PREDTOP_LIB=$L/libpredtop_$v.so timeout 120 python tools/repeat_check.py >> gpurun_out/rc.txt 2>&1; done
timeout 400 python -m pytest tests -m gpu -x -q > gpurun_out/pt.txt 2>&1
timeout 300 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --profile-json gpurun_out/prof_main.json > gpurun_out/bench_main.json 2>gpurun_out/bench_main.err
for v in "$@"; do
  PREDTOP_LIB=$L/libpredtop_$v.so timeout 300 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --profile-json gpurun_out/prof_$v.json > gpurun_out/bench_$v.json 2>gpurun_out/bench_$v.err
done
