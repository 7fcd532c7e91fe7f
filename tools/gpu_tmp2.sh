PREDTOP_LIB=$PWD/paper_conf_ipps_acharyas25_b200/lib/libpredtop_poly6.so timeout 300 python -m pytest tests -m gpu -q -x --timeout 100 -k "moe or tc or exact" 2>&1 | tail -1
bash tools/gpu_ab.sh poly4 poly6 poly8 2>&1 | grep -v "^$"
