#!/bin/bash
# C2 StringMatch Map shape sweep (map warps, super-window size), then one ncu capture of the C2 Map.
mkdir -p gpurun_out
B="python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep13.jsonl
for v in "C2 X=0" "C2 BMR_MAP_PF=0" "C2 BMR_MAP_PF=1" "C2 BMR_MAP_PF=4"; do
  set -- $v
  echo "{\"sweep\": \"$v\"}" >> gpurun_out/sweep13.jsonl
  env $2 timeout 300 $B --workload $1 >> gpurun_out/sweep13.jsonl 2>> gpurun_out/sweep13.err
done
BMR_LIB=variants/libbmr_sm12.so timeout 120 true
timeout 300 python -m pytest tests -m gpu -x -q -k sm > gpurun_out/sm_tests.log 2>&1; echo rc=$? >> gpurun_out/sm_tests.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_map -c 1 -o gpurun_out/e_C2_k_map -f python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline --workload C2 > gpurun_out/ncu_C2.log 2>&1
