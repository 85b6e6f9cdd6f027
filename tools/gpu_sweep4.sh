#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/gpu_tests.log
B="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep4.jsonl
for w in C4 C5 C2; do for h in 0 2; do
  echo "{\"sweep\": \"$w wait=$h\"}" >> gpurun_out/sweep4.jsonl
  BMR_MAP_WAIT=$h timeout 300 $B --workload $w >> gpurun_out/sweep4.jsonl 2>> gpurun_out/sweep4.err
done; done
