#!/bin/bash
O=gpurun_out; mkdir -p $O
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize.py > $O/sanitize_$tool.txt 2>&1
  echo "$tool rc=$?" >> $O/sanitize_$tool.txt
  tail -4 $O/sanitize_$tool.txt
done
