#!/bin/bash
# WordCount combiner table size (2^13 slots; output buffers 8 KB, 640 staged offsets to make room)
mkdir -p gpurun_out
BMR_LIB=variants/libbmr_comb13.so timeout 300 python -m pytest tests -m gpu -x -q -k "wc" > gpurun_out/wc_tests_comb13.log 2>&1; echo "rc=$?" >> gpurun_out/wc_tests_comb13.log
B="python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep17.jsonl
for v in "C5 X=0" "C5 BMR_LIB=variants/libbmr_out8.so" "C5 BMR_LIB=variants/libbmr_comb13.so" "C1 X=0" "C1 BMR_LIB=variants/libbmr_comb13.so"; do
  set -- $v
  echo "{\"sweep\": \"$v\"}" >> gpurun_out/sweep17.jsonl
  env $2 timeout 300 $B --workload $1 >> gpurun_out/sweep17.jsonl 2>> gpurun_out/sweep17.err
done
