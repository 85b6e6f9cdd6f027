#!/bin/bash
# Round-2 start: GPU suite, C5 bench, ncu --set full (source) of the C5 WordCount Map kernel.
O=gpurun_out/r02a; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt 2>&1
timeout 600 python -m pytest tests -m gpu -x -q > $O/gpu_tests.log 2>&1; echo "rc=$?" >> $O/gpu_tests.log
timeout 300 python bench.py --steps 5 --warmup 3 > $O/bench_C5.json 2> $O/bench_C5.err
B="python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_map -c 1 -o $O/C5_k_map -f $B --workload C5 > $O/ncu_C5.log 2>&1
ls -la $O
