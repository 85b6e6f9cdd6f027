#!/bin/bash
# ncu --set full captures of the current top kernels (one GPU): C5 Map, C5 u32 onesweep, C2 Map.
set -x
mkdir -p gpurun_out
B="python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline"
N="ncu --set full --clock-control none --import-source on"
timeout 900 $N -k regex:k_map -c 1 -o gpurun_out/c_C5_k_map -f $B --workload C5 > gpurun_out/ncu_C5a.log 2>&1
timeout 900 $N -k regex:'k_onesweep<unsigned int' -c 1 -o gpurun_out/c_C5_os32 -f $B --workload C5 > gpurun_out/ncu_C5b.log 2>&1
timeout 600 $N -k regex:k_map -c 1 -o gpurun_out/c_C2_k_map -f $B --workload C2 > gpurun_out/ncu_C2.log 2>&1
ls -la gpurun_out/
