timeout 300 python -m pytest tests -m gpu -q -x --timeout 100 -k "moe or exact or tc or mixed or invalid" > gpurun_out/pt_ab.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pt_ab.txt; tail -3 gpurun_out/pt_ab.txt
grep -E "FAILED|Error" gpurun_out/pt_ab.txt | head -5
timeout 200 python bench.py --config moe --no-cpu-baseline --no-also --steps 20 > gpurun_out/bench_p.json 2>gpurun_out/bench_p.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_p.json').read().strip().splitlines()[-1]); print('persist', round(d['value']), {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items() if v['ms_per_step']>0.3})" || tail -3 gpurun_out/bench_p.err
PREDTOP_ATTN_PERSIST=0 timeout 200 python bench.py --config moe --no-cpu-baseline --no-also --steps 20 > gpurun_out/bench_np.json 2>gpurun_out/bench_np.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_np.json').read().strip().splitlines()[-1]); print('nonpersist', round(d['value']), {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items() if v['ms_per_step']>0.3})" || tail -3 gpurun_out/bench_np.err
