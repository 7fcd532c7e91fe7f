timeout 400 python -m pytest tests -m gpu -q -x --timeout 200 -k "dag or hops or moe or 16k" > gpurun_out/pt_ab.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pt_ab.txt; tail -3 gpurun_out/pt_ab.txt
grep -E "FAILED|Error" gpurun_out/pt_ab.txt | head -5
for c in moe 16k; do
timeout 200 python bench.py --config $c --no-cpu-baseline --no-also --steps 10 > gpurun_out/bench_$c.json 2>gpurun_out/bench_$c.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_$c.json').read().strip().splitlines()[-1]); print('$c', round(d['value'],1), {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items() if v['ms_per_step']>0.1})" || tail -3 gpurun_out/bench_$c.err
done
