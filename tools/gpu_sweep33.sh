#!/bin/bash
mkdir -p gpurun_out
timeout 400 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "rc=$?" >> gpurun_out/gpu_tests.log
B="python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep33.jsonl
for v in "C5 X=0" "C5 BMR_SEG_TWO_PASS=1"; do
  set -- $v
  echo "{\"sweep\": \"$v\"}" >> gpurun_out/sweep33.jsonl
  env $2 timeout 300 $B --workload $1 >> gpurun_out/sweep33.jsonl 2>> gpurun_out/sweep33.err
done
