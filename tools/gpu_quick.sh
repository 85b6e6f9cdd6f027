#!/bin/bash
# Quick GPU check: parity tests + C5 bench line.
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/gpu_tests.log
for w in ${WORKLOADS:-C5}; do
  timeout 600 python bench.py --workload $w --steps 5 --warmup 3 ${BENCH_ARGS} > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
done
