#!/bin/bash
mkdir -p gpurun_out
N="ncu --set full --clock-control none --import-source on"
P="python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline"
timeout 600 $N -k regex:k_map -c 1 -o gpurun_out/full4_C5_k_map -f $P --workload C5 > /dev/null 2>&1
timeout 600 $N -k regex:"k_onesweep<unsigned int" -s 2 -c 1 -o gpurun_out/full4_C5_os32 -f $P --workload C5 > /dev/null 2>&1
timeout 600 $N -k regex:"k_hist|k_seg_count" -c 4 -o gpurun_out/full4_C5_misc -f $P --workload C5 > /dev/null 2>&1
timeout 600 $N -k regex:k_map -c 1 -o gpurun_out/full4_C2_k_map -f $P --workload C2 > /dev/null 2>&1
timeout 600 $N -k regex:k_map -c 1 -o gpurun_out/full4_C3_k_map -f $P --workload C3 > /dev/null 2>&1
timeout 600 $N -k regex:k_map -c 1 -o gpurun_out/full4_C4_k_map -f $P --workload C4 > /dev/null 2>&1
