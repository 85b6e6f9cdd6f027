#!/bin/bash
# Parameter sweep (one GPU): Map L2 prefetch distance, u32 sort variants.  One JSON line each.
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/gpu_tests.log
B="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep.jsonl
for pf in 0 2 4 8; do
  echo "{\"sweep\": \"C2 pf=$pf\"}" >> gpurun_out/sweep.jsonl
  BMR_MAP_PF=$pf timeout 300 $B --workload C2 >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err
done
for pf in 0 4; do
  echo "{\"sweep\": \"C4 pf=$pf\"}" >> gpurun_out/sweep.jsonl
  BMR_MAP_PF=$pf timeout 300 $B --workload C4 >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err
done
for v in 0 1 2 3; do
  echo "{\"sweep\": \"C5 var32=$v\"}" >> gpurun_out/sweep.jsonl
  BMR_SORT_VARIANT32=$v timeout 300 $B --workload C5 >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err
done
echo "{\"sweep\": \"C5 cfg=1\"}" >> gpurun_out/sweep.jsonl
BMR_SORT_CFG=1 timeout 300 $B --workload C5 >> gpurun_out/sweep.jsonl 2>> gpurun_out/sweep.err
