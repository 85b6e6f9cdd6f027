#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/gpu_tests.log
B="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep8.jsonl
for v in "C5 BMR_SORT_VARIANT32=2" "C5 BMR_SORT_VARIANT32=20" "C5 BMR_SORT_VARIANT32=21" "C4 X=0" "C2 X=0"; do
  set -- $v
  echo "{\"sweep\": \"$v\"}" >> gpurun_out/sweep8.jsonl
  env $2 timeout 300 $B --workload $1 >> gpurun_out/sweep8.jsonl 2>> gpurun_out/sweep8.err
done
