#!/bin/bash
mkdir -p gpurun_out
B="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep7.jsonl
for v in "C5 BMR_SORT_VARIANT32=2" "C5 BMR_SORT_VARIANT32=18" "C5 BMR_SORT_VARIANT32=19" "C5 BMR_MAP_WAIT=2"; do
  set -- $v
  echo "{\"sweep\": \"$v\"}" >> gpurun_out/sweep7.jsonl
  env $2 timeout 300 $B --workload $1 >> gpurun_out/sweep7.jsonl 2>> gpurun_out/sweep7.err
done
