#!/bin/bash
mkdir -p gpurun_out/final
O=gpurun_out/final
timeout 300 python bench.py --workload C2 --steps 5 --warmup 3 > $O/bench_C2.json 2> $O/bench_C2.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_map -c 1 -o $O/r01_C2_k_map -f python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline --workload C2 > $O/ncu_C2.log 2>&1
