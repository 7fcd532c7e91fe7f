timeout 300 python -m pytest tests -m gpu -q -x --timeout 100 -k "moe or tc or exact" 2>&1 | tail -1
bash tools/gpu_ab.sh oldattn 2>&1 | grep -v "^$"
bash tools/gpu_ab.sh oldattn 2>&1 | grep -v "^$" | tail -2
