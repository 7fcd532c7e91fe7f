timeout 400 python -m pytest tests -m gpu -q -x --timeout 90 -k "moe or tc or tiny or exact" > gpurun_out/pt_attn.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pt_attn.txt; tail -3 gpurun_out/pt_attn.txt
timeout 240 python bench.py --config moe --no-cpu-baseline --no-also --steps 20 > gpurun_out/bench_moe.json 2>gpurun_out/bench_moe.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_moe.json').read().strip().splitlines()[-1]); print(d['value'], d['kernels']['attention']['ms_per_step'], d['roofline']['frac'])"
PREDTOP_LIB=$PWD/paper_conf_ipps_acharyas25_b200/lib/libpredtop_trace.so timeout 120 python tools/attn_trace.py moe > gpurun_out/attn_trace.txt 2>&1; tail -12 gpurun_out/attn_trace.txt
