#!/bin/bash
# WordCount long-word queue across windows: WC parity (+ memory modes), C5 with / without
mkdir -p gpurun_out
timeout 300 python -m pytest tests -m gpu -x -q -k "wc or memory_modes or fullsize or host_lines" > gpurun_out/wc_tests_lq.log 2>&1; echo "rc=$?" >> gpurun_out/wc_tests_lq.log
B="python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep18.jsonl
for v in "C5 X=0" "C5 BMR_LIB=variants/libbmr_lq0.so"; do
  set -- $v
  echo "{\"sweep\": \"$v\"}" >> gpurun_out/sweep18.jsonl
  env $2 timeout 300 $B --workload $1 >> gpurun_out/sweep18.jsonl 2>> gpurun_out/sweep18.err
done
