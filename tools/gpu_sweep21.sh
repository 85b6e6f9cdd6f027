#!/bin/bash
# KMeans points per map lane: parity (default 2), C3 with 1 / 2 / 4
mkdir -p gpurun_out
timeout 300 python -m pytest tests -m gpu -x -q -k "km or memory_modes" > gpurun_out/km_tests.log 2>&1; echo "rc=$?" >> gpurun_out/km_tests.log
BMR_LIB=variants/libbmr_ppl4.so timeout 300 python -m pytest tests -m gpu -x -q -k "km" > gpurun_out/km_tests4.log 2>&1; echo "rc=$?" >> gpurun_out/km_tests4.log
B="python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep21.jsonl
for v in "C3 X=0" "C3 BMR_LIB=variants/libbmr_ppl1.so" "C3 BMR_LIB=variants/libbmr_ppl4.so"; do
  set -- $v
  echo "{\"sweep\": \"$v\"}" >> gpurun_out/sweep21.jsonl
  env $2 timeout 300 $B --workload $1 >> gpurun_out/sweep21.jsonl 2>> gpurun_out/sweep21.err
done
