#!/bin/bash
# Full-size ncu --set full captures of the top kernels (one GPU), round 1 refresh.
set -x
B="python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline"
N="ncu --set full --clock-control none --import-source on"
timeout 900 $N -k regex:k_map -c 1 -o gpurun_out/full_C5_k_map -f $B --workload C5 > gpurun_out/ncu_C5a.log 2>&1
timeout 900 $N -k regex:k_onesweep -c 2 -o gpurun_out/full_C5_k_onesweep -f $B --workload C5 > gpurun_out/ncu_C5b.log 2>&1
timeout 600 $N -k regex:k_map -c 1 -o gpurun_out/full_C2_k_map -f $B --workload C2 > gpurun_out/ncu_C2.log 2>&1
timeout 600 $N -k regex:'k_map|k_reduce_km|k_onesweep' -c 4 -o gpurun_out/full_C3 -f $B --workload C3 > gpurun_out/ncu_C3.log 2>&1
timeout 600 $N -k regex:'k_map|k_seg_count' -c 2 -o gpurun_out/full_C4 -f $B --workload C4 > gpurun_out/ncu_C4.log 2>&1
ls -la gpurun_out/
