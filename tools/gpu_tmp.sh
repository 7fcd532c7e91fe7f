timeout 300 python -m pytest tests -m gpu -q -x --timeout 100 -k "moe or unfused or taps" > gpurun_out/pt_ab.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pt_ab.txt; tail -2 gpurun_out/pt_ab.txt
grep -E "FAILED|Error" gpurun_out/pt_ab.txt | head -3
timeout 200 python bench.py --config moe --no-cpu-baseline --no-also --steps 20 > gpurun_out/bench_moe.json 2>gpurun_out/bench_moe.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_moe.json').read().strip().splitlines()[-1]); print(round(d['value']), {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items() if v['ms_per_step']>0.3})" || tail -3 gpurun_out/bench_moe.err
PREDTOP_LIB=$PWD/paper_conf_ipps_acharyas25_b200/lib/libpredtop_trace.so timeout 120 python tools/l256_trace.py > gpurun_out/l256_trace3.txt 2>&1; sed -n 1,8p gpurun_out/l256_trace3.txt
