#!/bin/bash
mkdir -p gpurun_out
B="python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --workload C4"
: > gpurun_out/sweep26.jsonl
timeout 300 $B >> gpurun_out/sweep26.jsonl 2>> gpurun_out/sweep26.err
timeout 300 $B --xchg fused >> gpurun_out/sweep26.jsonl 2>> gpurun_out/sweep26.err
