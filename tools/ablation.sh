#!/bin/bash
# the paper's memory-usage modes (SIO / SO / SI / G, Fig. 5)
# on the same Map kernel, every config, one GPU.  One JSON line per (config, mode).
mkdir -p gpurun_out
B="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/ablation.jsonl
for w in C5 C2 C3 C4; do for m in SIO SO SI G; do for c in "" "--no-map-combine"; do
  if [ "$w" = "C2" ] || [ "$w" = "C4" ]; then [ -n "$c" ] && continue; fi
  timeout 300 $B --workload $w --mode $m $c >> gpurun_out/ablation.jsonl 2>> gpurun_out/ablation.err
done; done; done
