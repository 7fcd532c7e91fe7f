timeout 300 python -m pytest tests -m gpu -q -x --timeout 200 -k "16k or large_path or dag" > gpurun_out/pt_ab.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/pt_ab.txt; tail -2 gpurun_out/pt_ab.txt
grep -E "FAILED|Error" gpurun_out/pt_ab.txt | head -3
for v in default ra16 ra4; do
  if [ "$v" != default ]; then export PREDTOP_LIB=$PWD/paper_conf_ipps_acharyas25_b200/lib/libpredtop_$v.so; else unset PREDTOP_LIB; fi
  timeout 200 python bench.py --config 16k --no-cpu-baseline --no-also --steps 10 > gpurun_out/b16_$v.json 2>gpurun_out/b16_$v.err
  python -c "
import json; d=json.loads(open('gpurun_out/b16_$v.json').read().strip().splitlines()[-1]); print('$v', round(d['value'],1), {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items() if v['ms_per_step']>0.1})" || tail -3 gpurun_out/b16_$v.err
done
