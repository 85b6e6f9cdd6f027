#!/bin/bash
mkdir -p gpurun_out
: > gpurun_out/sort_bench.txt
for z in 1 0; do for v in 2 66 130 258 386 194 322; do
  echo "== variant $v zipf $z" >> gpurun_out/sort_bench.txt
  BMR_SORT_VARIANT32=$v timeout 120 tools/micro/sort_bench 672 30 $z >> gpurun_out/sort_bench.txt 2>&1
done; done
