#!/bin/bash
mkdir -p gpurun_out
B="python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep32.jsonl
for v in "C5 X=0" "C5 BMR_SORT_CFG=1" "C5 BMR_SORT_CFG=2" "C5 BMR_SORT_CFG=3" "C5 BMR_SORT_ADAPT=20" "C5 BMR_SORT_ADAPT=28"; do
  set -- $v
  echo "{\"sweep\": \"$v\"}" >> gpurun_out/sweep32.jsonl
  env $2 timeout 300 $B --workload $1 >> gpurun_out/sweep32.jsonl 2>> gpurun_out/sweep32.err
done
