#!/bin/bash
# full GPU tests + smoke + C5/C4 bench lines (quick validation of the current defaults)
mkdir -p gpurun_out/check
O=gpurun_out/check
timeout 400 python -m pytest tests -m gpu -x -q > $O/gpu_tests.log 2>&1; echo "rc=$?" >> $O/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1
for w in ${WORKLOADS:-C5 C4}; do
  timeout 300 python bench.py --workload $w --steps 5 --warmup 3 > $O/bench_$w.json 2> $O/bench_$w.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_C4.csv python bench.py --workload C4 --steps 2 --warmup 1 --no-cpu-baseline --e2e-steps 0 > $O/ncu_launch.log 2>&1
