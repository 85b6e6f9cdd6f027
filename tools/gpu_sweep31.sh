#!/bin/bash
mkdir -p gpurun_out
timeout 400 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "rc=$?" >> gpurun_out/gpu_tests.log
B="python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep31.jsonl
for w in C5 C4; do timeout 300 $B --workload $w >> gpurun_out/sweep31.jsonl 2>> gpurun_out/sweep31.err; done
