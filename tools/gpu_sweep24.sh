#!/bin/bash
mkdir -p gpurun_out
timeout 300 python -m pytest tests -m gpu -x -q -k "wc or sort" > gpurun_out/wc_tests_hist.log 2>&1; echo "rc=$?" >> gpurun_out/wc_tests_hist.log
timeout 300 python bench.py --workload C5 --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/bench_C5_hist.json 2> gpurun_out/bench_C5_hist.err
