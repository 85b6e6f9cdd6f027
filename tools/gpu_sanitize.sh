#!/bin/bash
mkdir -p gpurun_out
for t in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $t --print-limit 20 python tools/sanitize_small.py > gpurun_out/sanitize_$t.log 2>&1
  echo "rc=$?" >> gpurun_out/sanitize_$t.log
done
