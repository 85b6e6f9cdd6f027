#!/bin/bash
# Round-1 evidence refresh: tests, smoke, bench lines (all configs + reference arm), C5 launch
# list, ncu --set full of every config's Map and of one C5 u32 onesweep pass.
set -x
mkdir -p gpurun_out/final
O=gpurun_out/final
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt 2>&1
timeout 400 python -m pytest tests -m gpu -x -q > $O/gpu_tests.log 2>&1; echo "rc=$?" >> $O/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1
for w in C5 C2 C3 C4; do
  timeout 600 python bench.py --workload $w --steps 5 --warmup 3 > $O/bench_$w.json 2> $O/bench_$w.err
done
timeout 300 python bench.py --impl reference --steps 2 --warmup 3 > $O/bench_reference_C5.json 2> $O/bench_reference_C5.err
timeout 300 python bench.py --workload C4 --xchg fused --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench_C4_fused_xchg.json 2> $O/bench_C4_fused.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_C5.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --e2e-steps 0 > $O/ncu_launch.log 2>&1
B="python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline"
N="ncu --set full --clock-control none --import-source on"
for w in C5 C2 C3 C4; do
  timeout 900 $N -k regex:k_map -c 1 -o $O/r01_${w}_k_map -f $B --workload $w > $O/ncu_$w.log 2>&1
done
timeout 600 $N --kernel-name-base demangled -k "regex:k_onesweep<unsigned int" -c 1 -o $O/r01_C5_os32 -f $B --workload C5 > $O/ncu_os32.log 2>&1
ls -la $O
