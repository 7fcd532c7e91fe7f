# GEMM epilogue (32-column steps) check: forward/unfused gpu tests, MoE + GPT bench x2
O=gpurun_out; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 -k "forward or unfused or moe or gemm or tap" > $O/pt_g.txt 2>&1; echo "pytest rc=$?"; tail -1 $O/pt_g.txt
for c in moe gpt moe gpt; do
  timeout 240 python bench.py --config $c --no-cpu-baseline --no-also --steps 20 > $O/bench_e.json 2>$O/bench_e.err
  python -c "
import json; d=json.loads(open('$O/bench_e.json').read().strip().splitlines()[-1]); print('$c', round(d['value'],1), {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items() if k in ('gemm_qkv','attention','layer_tail')})" || tail -3 $O/bench_e.err
done
