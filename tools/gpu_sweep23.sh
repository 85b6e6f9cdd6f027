#!/bin/bash
mkdir -p gpurun_out
B="python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep23.jsonl
for v in "C4 X=0" "C4 BMR_MAP_WAIT=1" "C4 BMR_MAP_WAIT=2" "C5 X=0" "C5 BMR_MAP_WAIT=1" "C5 BMR_MAP_WAIT=2"; do
  set -- $v
  echo "{\"sweep\": \"$v\"}" >> gpurun_out/sweep23.jsonl
  env $2 timeout 300 $B --workload $1 >> gpurun_out/sweep23.jsonl 2>> gpurun_out/sweep23.err
done
