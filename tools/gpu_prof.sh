#!/bin/bash
# tests + C2/C5/C4 bench A/B + ncu full captures of the Map kernels (one GPU)
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/gpu_tests.log
B="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep5.jsonl
for v in "C2 BMR_MAP_DYN=0" "C2 BMR_MAP_DYN=1" "C2 BMR_MAP_PF=2" "C5 X=0" "C4 X=0"; do
  set -- $v
  echo "{\"sweep\": \"$v\"}" >> gpurun_out/sweep5.jsonl
  env $2 timeout 300 $B --workload $1 >> gpurun_out/sweep5.jsonl 2>> gpurun_out/sweep5.err
done
N="ncu --set full --clock-control none --import-source on"
P="python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline"
timeout 600 $N -k regex:k_map -c 1 -o gpurun_out/full3_C5_k_map -f $P --workload C5 > /dev/null 2>&1
timeout 600 $N -k regex:k_map -c 1 -o gpurun_out/full3_C2_k_map -f $P --workload C2 > /dev/null 2>&1
timeout 600 $N -k regex:k_map -c 1 -o gpurun_out/full3_C4_k_map -f $P --workload C4 > /dev/null 2>&1
