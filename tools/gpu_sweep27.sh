#!/bin/bash
mkdir -p gpurun_out
timeout 300 python -m pytest tests -m gpu -x -q -k "ii or multirank or wc_multi" > gpurun_out/gpu_tests.log 2>&1; echo "rc=$?" >> gpurun_out/gpu_tests.log
B="python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --workload C4"
: > gpurun_out/sweep27.jsonl
timeout 300 $B >> gpurun_out/sweep27.jsonl 2>> gpurun_out/sweep27.err
timeout 300 $B --xchg fused >> gpurun_out/sweep27.jsonl 2>> gpurun_out/sweep27.err
timeout 300 python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --workload C5 >> gpurun_out/sweep27.jsonl 2>> gpurun_out/sweep27.err
