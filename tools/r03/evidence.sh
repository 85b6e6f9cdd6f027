#!/bin/bash
# Round-2 evidence (second session): GPU suite, smoke, bench lines of every config (+ reference
# arm, strong scaling, literal order, KM full scan, memory-mode ablations), C5 / C4 / C3 launch
# lists, ncu --set full exports (CSV pages) of every config's Map and of C4's onesweep pass.
O=gpurun_out/${TAG:-ev3}; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt 2>&1
lscpu > $O/lscpu.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q > $O/gpu_tests.log 2>&1; echo "rc=$?" >> $O/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1
for w in C5 C4 C3 C2 C1; do
  timeout 600 python bench.py --workload $w --steps 10 --warmup 3 > $O/bench_$w.json 2> $O/bench_$w.err
done
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_reference_C5.json 2> $O/bench_reference_C5.err
timeout 900 python bench.py --scaling strong --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench_C5_strong_n1.json 2> $O/bench_C5_strong.err
timeout 600 python bench.py --no-map-combine --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench_C5_literal.json 2> $O/bench_C5_literal.err
timeout 600 python bench.py --workload C3 --km-full-scan --steps 10 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench_C3_full_scan.json 2> $O/bench_C3_full_scan.err
for m in SO SI G; do for w in C5 C4 C3 C2; do
  timeout 600 python bench.py --workload $w --mode $m --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/abl_${w}_$m.json 2> $O/abl_${w}_$m.err
done; done
B="python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline"
for w in C5 C4 C3; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$w.csv $B --workload $w > /dev/null 2>&1
done
for w in C5 C4 C3 C2; do TAG=${TAG:-ev3} NAME=${w}_map K=k_map WL=$w bash tools/r03/ncu_export.sh > /dev/null 2>&1; done
TAG=${TAG:-ev3} NAME=C4_onesweep K=k_onesweep S=2 WL=C4 bash tools/r03/ncu_export.sh > /dev/null 2>&1
TAG=${TAG:-ev3} NAME=C5_xtab K=k_xtab_extract WL=C5 bash tools/r03/ncu_export.sh > /dev/null 2>&1
ls -la $O | head -80
