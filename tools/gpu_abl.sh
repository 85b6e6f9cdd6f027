#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/gpu_tests.log
bash tools/ablation.sh
N="ncu --set full --clock-control none --import-source on"
P="python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline"
timeout 600 $N -k regex:k_onesweep -c 1 -o gpurun_out/full4_C5_os32 -f $P --workload C5 > gpurun_out/ncu_os.log 2>&1
