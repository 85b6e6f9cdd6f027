#!/bin/bash
mkdir -p gpurun_out
B="python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep30.jsonl
for v in "C3 X=0" "C3 BMR_LIB=variants/libbmr_kmu16.so" "C3 X=1"; do
  set -- $v
  echo "{\"sweep\": \"$v\"}" >> gpurun_out/sweep30.jsonl
  env $2 timeout 300 $B --workload $1 >> gpurun_out/sweep30.jsonl 2>> gpurun_out/sweep30.err
done
