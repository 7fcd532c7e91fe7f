# A/B of the working tree (default) against HEAD (libpredtop_head.so): dag tests on the default, MoE + 16k benches x2
O=gpurun_out; mkdir -p $O
true
for i in 1 2; do
for v in default head; do
  if [ "$v" != default ]; then export PREDTOP_LIB=$PWD/paper_conf_ipps_acharyas25_b200/lib/libpredtop_$v.so; else unset PREDTOP_LIB; fi
  for c in moe; do
  timeout 240 python bench.py --config $c --no-cpu-baseline --no-also --steps 10 > $O/bench_$v.json 2>$O/bench_$v.err
  python -c "
import json; d=json.loads(open('$O/bench_$v.json').read().strip().splitlines()[-1]); print('$v $c', round(d['value'],1), {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items() if k in ('readout','embed','attention')})" || tail -3 $O/bench_$v.err
  done
done
done
