#!/bin/bash
# adaptive u32 ranking: calibration (sort_bench E per digit) + C5 thresholds + WC parity
mkdir -p gpurun_out
: > gpurun_out/sort_bench2.txt
for v in; do echo "== variant $v" >> gpurun_out/sort_bench2.txt; BMR_SORT_VARIANT32=$v timeout 120 tools/micro/sort_bench 672 30 1 >> gpurun_out/sort_bench2.txt 2>&1; done
timeout 300 python -m pytest tests -m gpu -x -q -k "wc" > gpurun_out/wc_tests_adapt.log 2>&1; echo "rc=$?" >> gpurun_out/wc_tests_adapt.log
B="python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep14.jsonl
for v in "C5 BMR_SORT_ADAPT=24" "C5 BMR_SORT_ADAPT=0"; do
  set -- $v
  echo "{\"sweep\": \"$v\"}" >> gpurun_out/sweep14.jsonl
  env $2 BMR_SORT_DEBUG=1 timeout 300 $B --workload $1 >> gpurun_out/sweep14.jsonl 2>> gpurun_out/sweep14_$2.err
done
