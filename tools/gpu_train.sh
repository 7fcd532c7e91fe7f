#!/bin/bash
O=gpurun_out; mkdir -p $O; rm -f $O/parity_log.jsonl
timeout 900 python -m pytest tests/test_gpu_train.py -q -x -s --timeout 600 > $O/pt_train.txt 2>&1; echo "pytest rc=$?" >> $O/pt_train.txt
tail -25 $O/pt_train.txt
