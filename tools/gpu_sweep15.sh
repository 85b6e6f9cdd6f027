#!/bin/bash
# WordCount combiner probes: parity with 2 probes, C5 1/2/4 probes
mkdir -p gpurun_out
timeout 300 python -m pytest tests -m gpu -x -q -k "wc" > gpurun_out/wc_tests_probe.log 2>&1; echo "rc=$?" >> gpurun_out/wc_tests_probe.log
B="python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline"
: > gpurun_out/sweep15.jsonl
for v in "C5 X=0" "C5 BMR_LIB=variants/libbmr_probe1.so" "C5 BMR_LIB=variants/libbmr_probe4.so"; do
  set -- $v
  echo "{\"sweep\": \"$v\"}" >> gpurun_out/sweep15.jsonl
  env $2 timeout 300 $B --workload $1 >> gpurun_out/sweep15.jsonl 2>> gpurun_out/sweep15.err
done
