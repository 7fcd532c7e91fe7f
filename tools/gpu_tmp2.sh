PREDTOP_LIB=$PWD/paper_conf_ipps_acharyas25_b200/lib/libpredtop_stg2.so timeout 200 python -m pytest tests -m gpu -q -x --timeout 100 -k "moe" 2>&1 | tail -1
bash tools/gpu_ab.sh stg2 2>&1 | grep -v "^$"
