#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/gpu_tests.log
B="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep9.jsonl
for v in "C5 BMR_WC_BAL=1" "C5 BMR_WC_BAL=0" "C1 BMR_WC_BAL=1"; do
  set -- $v
  echo "{\"sweep\": \"$v\"}" >> gpurun_out/sweep9.jsonl
  env $2 timeout 300 $B --workload $1 >> gpurun_out/sweep9.jsonl 2>> gpurun_out/sweep9.err
done
