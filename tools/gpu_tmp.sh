O=gpurun_out
for i in 1 2; do
for v in nat rdfs; do
 for c in moe gpt; do
  if [ $v = rdfs ]; then export PREDTOP_PROBE_RDFS=1; else unset PREDTOP_PROBE_RDFS; fi
  timeout 300 python bench.py --config $c --no-cpu-baseline --no-also --steps 20 > $O/ord_${v}_$c.json 2>$O/ord_${v}_$c.err
  python -c "
import json; d=json.loads(open('$O/ord_${v}_$c.json').read().strip().splitlines()[-1]); print('$v $c', round(d['value']), 'frac', round(d['roofline']['frac'],3), {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items() if v['ms_per_step']>0.1})" || tail -3 $O/ord_${v}_$c.err
 done
done
done
