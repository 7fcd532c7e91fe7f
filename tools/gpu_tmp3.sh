# A/B of the working tree (default) against HEAD (libpredtop_head.so): dag tests on the default, MoE bench x2
O=gpurun_out; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 -k "dag or hops or prune or moe or search" > $O/pt_new.txt 2>&1; echo "pytest rc=$?"; tail -1 $O/pt_new.txt
for i in 1 2; do
for v in default head; do
  if [ "$v" != default ]; then export PREDTOP_LIB=$PWD/paper_conf_ipps_acharyas25_b200/lib/libpredtop_$v.so; else unset PREDTOP_LIB; fi
  timeout 240 python bench.py --config moe --no-cpu-baseline --no-also --steps 20 > $O/bench_$v.json 2>$O/bench_$v.err
  python -c "
import json; d=json.loads(open('$O/bench_$v.json').read().strip().splitlines()[-1]); print('$v', round(d['value'],1), {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items() if k.startswith('dag_') and v['ms_per_step']>0.1})" || tail -3 $O/bench_$v.err
done
done
