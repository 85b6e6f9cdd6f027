#!/bin/bash
mkdir -p gpurun_out/final
O=gpurun_out/final
for w in ${WORKLOADS:-C5}; do
  timeout 300 python bench.py --workload $w --steps 5 --warmup 3 > $O/bench_$w.json 2> $O/bench_$w.err
done
