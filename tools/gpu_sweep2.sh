#!/bin/bash
mkdir -p gpurun_out
B="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep2.jsonl
for w in C2 C5 C4 C3; do for h in 0 1; do
  echo "{\"sweep\": \"$w wait_hint=$h\"}" >> gpurun_out/sweep2.jsonl
  BMR_MAP_WAIT=$h timeout 300 $B --workload $w >> gpurun_out/sweep2.jsonl 2>> gpurun_out/sweep2.err
done; done
N="ncu --set full --clock-control none --import-source on"
timeout 600 $N -k regex:k_map -c 1 -o gpurun_out/full2_C2_k_map -f python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline --workload C2 > /dev/null 2>&1
timeout 900 $N -k regex:k_map -c 1 -o gpurun_out/full2_C5_k_map -f python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline --workload C5 > /dev/null 2>&1
