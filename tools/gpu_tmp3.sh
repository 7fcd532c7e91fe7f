PREDTOP_LIB=$PWD/paper_conf_ipps_acharyas25_b200/lib/libpredtop_pipe.so timeout 600 python -m pytest tests -m gpu -q -x --timeout 100 -k "moe or exact or tc" 2>&1 | tail -1
bash tools/gpu_ab.sh pipe 2>&1 | grep -v "^$" | tail -2
bash tools/gpu_ab.sh pipe 2>&1 | grep -v "^$" | tail -2
