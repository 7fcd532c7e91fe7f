# final build: the other BASELINE configs (16k, sweep, tiny) and the search NEXT row, default bench settings
O=gpurun_out; mkdir -p $O
for c in ${CFGS:-16k sweep tiny search}; do
  timeout 900 python bench.py --config $c > $O/bench_cfg_$c.json 2>$O/bench_cfg_$c.err; echo "$c rc=$?"
  python -c "
import json; d=json.loads(open('$O/bench_cfg_$c.json').read().strip().splitlines()[-1]); print('$c', round(d['value'],1), d['unit'], 'ms/step', round(d['ms_per_step'],3), 'e2e', d.get('e2e',{}).get('value'), 'frac', d.get('roofline',{}).get('frac'))" || tail -3 $O/bench_cfg_$c.err
done
