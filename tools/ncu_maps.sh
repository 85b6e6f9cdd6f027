#!/bin/bash
B="python bench.py --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_map -s 1 -c 1 -o gpurun_out/prof8_C4_k_map -f $B --workload C4 --units 512 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_map -s 1 -c 1 -o gpurun_out/prof8_C3_k_map -f $B --workload C3 --units 8388608 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_map -s 1 -c 1 -o gpurun_out/prof8_C2_k_map -f $B --workload C2 --units 512 > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_C5.csv $B --workload C5 > /dev/null 2>&1
ls gpurun_out | grep -E "prof8|launches"
