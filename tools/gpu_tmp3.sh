timeout 600 python -m pytest tests/test_gpu_dag.py -m gpu -q -x --timeout 300 2>&1 | tail -1
for v in default ra12 ra16; do
  if [ "$v" != default ]; then export PREDTOP_LIB=$PWD/paper_conf_ipps_acharyas25_b200/lib/libpredtop_$v.so; else unset PREDTOP_LIB; fi
  timeout 300 python bench.py --config 16k --no-cpu-baseline --no-also --steps 5 > gpurun_out/bench_16k_$v.json 2>gpurun_out/bench_16k.err
  python -c "
import json; d=json.loads(open('gpurun_out/bench_16k_$v.json').read().strip().splitlines()[-1]); print('$v', d['value'], d['ms_per_step'], {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items() if v['ms_per_step']>0.05})" || tail -3 gpurun_out/bench_16k.err
done
