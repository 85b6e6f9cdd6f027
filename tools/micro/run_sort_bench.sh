#!/bin/bash
# u32 keys-only onesweep passes, match.any vs shared-memory OR-mask ranking, Zipf and uniform keys
mkdir -p gpurun_out
: > gpurun_out/sort_bench.txt
for z in 1 0; do for r in 0 1; do
  echo "== rank $r zipf $z" >> gpurun_out/sort_bench.txt
  timeout 120 tools/micro/sort_bench 672 30 $z $r >> gpurun_out/sort_bench.txt 2>&1
done; done
