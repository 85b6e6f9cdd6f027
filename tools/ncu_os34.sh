#!/bin/bash
mkdir -p gpurun_out
BMR_SORT_VARIANT32=34 timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:k_onesweep<unsigned int" -s 2 -c 1 -o gpurun_out/c_C5_os34 -f python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline --workload C5 > gpurun_out/ncu_os34.log 2>&1
