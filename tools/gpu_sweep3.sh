#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/gpu_tests.log
B="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep3.jsonl
for w in C2 C5 C4; do for d in 0 1; do
  echo "{\"sweep\": \"$w dyn=$d\"}" >> gpurun_out/sweep3.jsonl
  BMR_MAP_DYN=$d timeout 300 $B --workload $w >> gpurun_out/sweep3.jsonl 2>> gpurun_out/sweep3.err
done; done
