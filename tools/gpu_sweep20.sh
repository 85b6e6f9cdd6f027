#!/bin/bash
mkdir -p gpurun_out
timeout 300 python -m pytest tests -m gpu -x -q -k "km or memory_modes" > gpurun_out/km_tests.log 2>&1; echo "rc=$?" >> gpurun_out/km_tests.log
timeout 300 python bench.py --workload C3 --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench_C3_km.json 2> gpurun_out/bench_C3_km.err
