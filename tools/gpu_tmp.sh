# d_h = 16 per-graph split between k_attn and the tcgen05 kernel: parity tests, split-size sweep on the search config, 16k and GPT
O=gpurun_out; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -q -x --timeout 300 -k "forward or 16k or search or hops or tc or moe or attention" > $O/pt_new.txt 2>&1; echo "pytest rc=$?"; tail -1 $O/pt_new.txt
run() {  # name, config, env...
  n=$1; c=$2; shift 2
  env "$@" timeout 600 python bench.py --config $c --no-cpu-baseline --no-also --steps 10 > $O/bench_$n.json 2>$O/bench_$n.err
  python -c "
import json; d=json.loads(open('$O/bench_$n.json').read().strip().splitlines()[-1]); print('$n', round(d['value'],1), round(d['ms_per_step'],3), {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items() if k in ('attention','layer_tail')})" || tail -3 $O/bench_$n.err
}
run search_all_tc search PREDTOP_ATTN_TC=1
run search_384 search PREDTOP_ATTN_TC16_MIN=384
run search_768 search PREDTOP_ATTN_TC16_MIN=768
run search_1536 search PREDTOP_ATTN_TC16_MIN=1536
run search_kattn search PREDTOP_ATTN_TC=0
run k16_default 16k
run k16_kattn 16k PREDTOP_ATTN_TC=0
run gpt_default gpt
run moe_default moe
