#!/bin/bash
# Quick GPU check: parity tests (TESTK selects a subset first) + bench lines of $WORKLOADS.
mkdir -p gpurun_out
if [ -n "$TESTK" ]; then
  timeout 300 python -m pytest tests -m gpu -x -q -k "$TESTK" > gpurun_out/gpu_tests_k.log 2>&1
  rc=$?; echo "tests-k rc=$rc" >> gpurun_out/gpu_tests_k.log
  [ $rc -ne 0 ] && exit $rc
fi
timeout ${TEST_TIMEOUT:-400} python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
echo "tests rc=$?" >> gpurun_out/gpu_tests.log
for w in ${WORKLOADS:-C5}; do
  timeout 300 python bench.py --workload $w --steps 5 --warmup 3 ${BENCH_ARGS} > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
done
