#!/bin/bash
# full GPU tests + C2/C3 bench lines + ncu capture of the C4 (InvertedIndex) Map.
mkdir -p gpurun_out
timeout 400 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "rc=$?" >> gpurun_out/gpu_tests.log
for w in C2 C3; do
  timeout 300 python bench.py --workload $w --steps 5 --warmup 3 > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_map -c 1 -o gpurun_out/e_C4_k_map -f python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline --workload C4 > gpurun_out/ncu_C4.log 2>&1
