#!/bin/bash
# Round-2 evidence (third session): GPU suite, smoke, bench lines of every config (C5 with e2e and
# the CPU baseline), the reference arm, C5 strong scaling at N = 1, launch lists of C5 / C4, ncu
# exports of the C5 Map.
O=gpurun_out/${TAG:-ev4}; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q > $O/gpu_tests.log 2>&1; echo "rc=$?" >> $O/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1
for w in C5 C4 C3 C2 C1; do
  timeout 600 python bench.py --workload $w --steps 10 --warmup 3 > $O/bench_$w.json 2> $O/bench_$w.err
done
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_reference_C5.json 2> $O/bench_reference_C5.err
timeout 900 python bench.py --scaling strong --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench_C5_strong_n1.json 2> $O/bench_C5_strong.err
B="python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline"
for w in C5 C4; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$w.csv $B --workload $w > /dev/null 2>&1
done
TAG=${TAG:-ev4} NAME=C5_map K=k_map WL=C5 bash tools/r03/ncu_export.sh > /dev/null 2>&1
ls -la $O | head -60
