#!/bin/bash
# ncu evidence for round 1 (run under gpurun on one B200).  Launch list of one C5 step, plus
# full-set captures of the top kernels on a reduced (1 GiB) shard.
set -x
B="python bench.py --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_C5.csv $B --workload C5 > /dev/null 2>&1
for k in k_map k_onesweep k_seg_count k_reduce_wc_small k_reduce_wc_large k_hist; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$k -s 1 -c 1 -o gpurun_out/prof_C5_$k -f $B --workload C5 --units 1024 > /dev/null 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_map -c 1 -o gpurun_out/prof_C4_k_map -f $B --workload C4 --units 512 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_map -c 1 -o gpurun_out/prof_C2_k_map -f $B --workload C2 --units 512 > /dev/null 2>&1
ls -la gpurun_out/
