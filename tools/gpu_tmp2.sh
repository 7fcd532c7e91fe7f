timeout 900 python -m pytest tests/test_gpu_dag.py tests/test_gpu_hops.py tests/test_gpu_prune.py -m gpu -q -x --timeout 300 2>&1 | tail -2
timeout 300 python -m pytest tests -m gpu -q -x --timeout 200 -k "16k or moe or invalid" 2>&1 | tail -2
timeout 200 python bench.py --config moe --no-cpu-baseline --no-also --steps 20 > gpurun_out/bench_moe.json 2>gpurun_out/bench_moe.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_moe.json').read().strip().splitlines()[-1]); print(round(d['value']), {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items() if v['ms_per_step']>0.05})" || tail -3 gpurun_out/bench_moe.err
timeout 300 python bench.py --config 16k --no-cpu-baseline --no-also --steps 5 > gpurun_out/bench_16k.json 2>gpurun_out/bench_16k.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_16k.json').read().strip().splitlines()[-1]); print(d['value'], d['ms_per_step'], {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items() if v['ms_per_step']>0.05})" || tail -3 gpurun_out/bench_16k.err
