#!/bin/bash
# variants bench + one ncu of k_map per variant (duration / DRAM bytes)
O=gpurun_out/${TAG:-vn}; mkdir -p $O
W=${WL:-C5}
bash tools/r02/variants.sh "$@" | grep json
for v in default "$@"; do
  L=""; [ "$v" != default ] && L="BMR_LIB=variants/libbmr_$v.so"
  env $L timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none -k regex:k_map -c 1 python bench.py --workload $W --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline 2>/dev/null | grep -E "gpu__time|dram__bytes|inst_executed" | sed "s/^/$v /"
done
