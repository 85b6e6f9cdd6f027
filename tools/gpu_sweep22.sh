#!/bin/bash
# StringMatch fast path in every memory mode: SM parity + memory-mode tests, C2 SIO/SO/SI/G
mkdir -p gpurun_out
timeout 300 python -m pytest tests -m gpu -x -q -k "sm or memory_modes" > gpurun_out/sm_tests_modes.log 2>&1; echo "rc=$?" >> gpurun_out/sm_tests_modes.log
B="python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/ablation_sm.jsonl
for m in SIO SO SI G; do timeout 300 $B --workload C2 --mode $m >> gpurun_out/ablation_sm.jsonl 2>> gpurun_out/ablation_sm.err; done
