#!/bin/bash
mkdir -p gpurun_out
timeout 300 python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --workload C4 --xchg fused > gpurun_out/bench_C4_fused.json 2> gpurun_out/bench_C4_fused.err
