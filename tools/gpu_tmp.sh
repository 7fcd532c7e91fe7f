# k_mask2 grid order check: dag/hops/forward gpu tests, MoE bench x2, ncu DRAM of k_mask2
O=gpurun_out; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 -k "dag or hops or prune or moe or 16k" > $O/pt_dag.txt 2>&1; echo "pytest rc=$?"; tail -1 $O/pt_dag.txt
for c in moe moe; do
  timeout 240 python bench.py --config $c --no-cpu-baseline --no-also --steps 20 > $O/bench_e.json 2>$O/bench_e.err
  python -c "
import json; d=json.loads(open('$O/bench_e.json').read().strip().splitlines()[-1]); print('$c', round(d['value']), {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items() if k.startswith('dag') or k in ('embed','attention')})" || tail -3 $O/bench_e.err
done
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:k_mask2 -c 1 python bench.py --config moe --no-cpu-baseline --no-also --steps 1 --warmup 1 2>&1 | grep -E "k_mask2|dram__|gpu__time" | head
