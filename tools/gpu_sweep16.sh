#!/bin/bash
# II '<' window filter: II parity + memory modes, C4 bench
mkdir -p gpurun_out
timeout 300 python -m pytest tests -m gpu -x -q -k "ii or memory_modes or fullsize" > gpurun_out/ii_tests.log 2>&1; echo "rc=$?" >> gpurun_out/ii_tests.log
timeout 300 python bench.py --workload C4 --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench_C4_ii.json 2> gpurun_out/bench_C4_ii.err
