# embed check: forward/tap parity + MoE/GPT bench
O=gpurun_out; mkdir -p $O
timeout 600 python -m pytest tests -m gpu -q -x --timeout 200 -k "forward or embed or tap or train" > $O/pt_fwd.txt 2>&1; echo "pytest rc=$?"; tail -1 $O/pt_fwd.txt
for c in moe gpt moe gpt; do
  timeout 240 python bench.py --config $c --no-cpu-baseline --no-also --steps 20 > $O/bench_e.json 2>$O/bench_e.err
  python -c "
import json; d=json.loads(open('$O/bench_e.json').read().strip().splitlines()[-1]); print('$c', round(d['value']), {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items() if k in ('embed','readout','attention')})" || tail -3 $O/bench_e.err
done
