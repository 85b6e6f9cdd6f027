#!/bin/bash
mkdir -p gpurun_out
BMR_LIB=variants/libbmr_smdyn.so timeout 300 python -m pytest tests -m gpu -x -q -k "sm" > gpurun_out/sm_tests_dyn.log 2>&1; echo "rc=$?" >> gpurun_out/sm_tests_dyn.log
B="python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep19.jsonl
for v in "C2 X=0" "C2 BMR_LIB=variants/libbmr_smdyn.so" "C2 BMR_LIB=variants/libbmr_smdyn8.so" "C2 BMR_LIB=variants/libbmr_sub8.so"; do
  set -- $v
  echo "{\"sweep\": \"$v\"}" >> gpurun_out/sweep19.jsonl
  env $2 timeout 300 $B --workload $1 >> gpurun_out/sweep19.jsonl 2>> gpurun_out/sweep19.err
done
