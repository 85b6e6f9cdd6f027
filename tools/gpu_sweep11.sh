#!/bin/bash
# u32 onesweep ranking variants (ballot peers + leader atomics): WC parity per variant, then C5 bench.
mkdir -p gpurun_out
for v in 66; do
  BMR_SORT_VARIANT32=$v timeout 300 python -m pytest tests -m gpu -x -q -k "wc" > gpurun_out/wc_tests_v$v.log 2>&1
  echo "rc=$?" >> gpurun_out/wc_tests_v$v.log
done
B="python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep11.jsonl
for v in "C5 BMR_SORT_VARIANT32=2" "C5 BMR_SORT_VARIANT32=3" "C5 BMR_SORT_VARIANT32=66" "C5 BMR_SORT_VARIANT32=67" "C5 BMR_SORT_VARIANT32=69"; do
  set -- $v
  echo "{\"sweep\": \"$v\"}" >> gpurun_out/sweep11.jsonl
  env $2 timeout 300 $B --workload $1 >> gpurun_out/sweep11.jsonl 2>> gpurun_out/sweep11.err
done
