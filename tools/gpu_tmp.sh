timeout 300 python -m pytest tests -m gpu -q -x --timeout 120 -k "moe or unfused or taps" > gpurun_out/pt_attn.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pt_attn.txt; tail -3 gpurun_out/pt_attn.txt
timeout 240 python bench.py --config moe --no-cpu-baseline --no-also --steps 20 > gpurun_out/bench_moe.json 2>gpurun_out/bench_moe.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_moe.json').read().strip().splitlines()[-1]); print(d['value'], {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items()})"
tail -3 gpurun_out/bench_moe.err
timeout 300 ncu --set full --clock-control none --import-source on -k regex:k_layer_tail256 -s 2 -c 1 -o gpurun_out/tail256_v2 python bench.py --config moe --graphs 128 --steps 1 --warmup 1 --no-cpu-baseline --no-also --no-extras --eager > gpurun_out/ncu_tail.log 2>&1
