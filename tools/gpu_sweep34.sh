#!/bin/bash
mkdir -p gpurun_out
timeout 300 python -m pytest tests -m gpu -x -q -k "ii or multirank or ipc or fullsize" > gpurun_out/ii48_tests.log 2>&1; echo "rc=$?" >> gpurun_out/ii48_tests.log
timeout 300 python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --workload C4 > gpurun_out/bench_C4_48.json 2> gpurun_out/bench_C4_48.err
