#!/bin/bash
# C2 StringMatch stage count / L2 prefetch sweep, then an ncu capture of one u32 onesweep pass (C5).
mkdir -p gpurun_out
B="python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep10.jsonl
for v in "C2 X=0" "C2 BMR_LIB=variants/libbmr_sm8.so" "C2 BMR_LIB=variants/libbmr_sm10.so" "C2 BMR_MAP_PF=2" "C2 BMR_MAP_PF=4" "C2 BMR_MAP_WAIT=1"; do
  set -- $v
  echo "{\"sweep\": \"$v\"}" >> gpurun_out/sweep10.jsonl
  env $2 timeout 300 $B --workload $1 >> gpurun_out/sweep10.jsonl 2>> gpurun_out/sweep10.err
done
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:k_onesweep<unsigned int" -c 1 -o gpurun_out/c_C5_os32 -f python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline --workload C5 > gpurun_out/ncu_os32.log 2>&1
