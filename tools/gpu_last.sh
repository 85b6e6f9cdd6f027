#!/bin/bash
mkdir -p gpurun_out/final
timeout 400 python -m pytest tests -m gpu -x -q > gpurun_out/final/gpu_tests.log 2>&1; echo "rc=$?" >> gpurun_out/final/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final/smoke.log 2>&1
timeout 300 python bench.py --steps 3 --warmup 3 > gpurun_out/final/bench_default.json 2> gpurun_out/final/bench_default.err
