# closure division check: dag/hops/moe/16k gpu tests, MoE bench x2, 16k bench
O=gpurun_out; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 -k "dag or hops or prune or moe or 16k" > $O/pt_dag.txt 2>&1; echo "pytest rc=$?"; tail -1 $O/pt_dag.txt
for c in moe moe 16k; do
  timeout 240 python bench.py --config $c --no-cpu-baseline --no-also --steps 20 > $O/bench_e.json 2>$O/bench_e.err
  python -c "
import json; d=json.loads(open('$O/bench_e.json').read().strip().splitlines()[-1]); print('$c', round(d['value'],1), {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items() if k.startswith('dag') or k in ('embed','attention')})" || tail -3 $O/bench_e.err
done
