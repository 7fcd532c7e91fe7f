# round-2 final ncu captures (one launch per hot kernel, --set full) for MoE and GPT
O=gpurun_out; mkdir -p $O
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_attn_tc|k_layer_tail256" -c 2 -o $O/final_moe2 python bench.py --config moe --no-cpu-baseline --no-also --steps 1 --warmup 1 > $O/ncu_final_moe2.log 2>&1; echo "moe rc=$?"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_layer_tail2" -c 1 -o $O/final_gpt2 python bench.py --config gpt --no-cpu-baseline --no-also --steps 1 --warmup 1 > $O/ncu_final_gpt2.log 2>&1; echo "gpt rc=$?"
