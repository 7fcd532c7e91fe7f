PREDTOP_LIB=$PWD/paper_conf_ipps_acharyas25_b200/lib/libpredtop_trace.so timeout 120 python tools/l256_trace.py > gpurun_out/l256_trace.txt 2>&1; sed -n 18,80p gpurun_out/l256_trace.txt
