#!/bin/bash
# full GPU tests, WC parity with the ballot ranking, C5 sort variants, C2.
mkdir -p gpurun_out
timeout 400 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "rc=$?" >> gpurun_out/gpu_tests.log
BMR_SORT_VARIANT32=34 timeout 300 python -m pytest tests -m gpu -x -q -k "wc" > gpurun_out/wc_tests_v34.log 2>&1; echo "rc=$?" >> gpurun_out/wc_tests_v34.log
B="python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep12.jsonl
for v in "C5 BMR_SORT_VARIANT32=2" "C5 BMR_SORT_VARIANT32=34" "C5 BMR_SORT_VARIANT32=35" "C2 BMR_MAP_PF=2" "C4 X=0"; do
  set -- $v
  echo "{\"sweep\": \"$v\"}" >> gpurun_out/sweep12.jsonl
  env $2 timeout 300 $B --workload $1 >> gpurun_out/sweep12.jsonl 2>> gpurun_out/sweep12.err
done
