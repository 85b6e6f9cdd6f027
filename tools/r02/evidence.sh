#!/bin/bash
# Round-2 evidence: GPU suite, smoke, bench lines of every config (+ reference arm, strong scaling,
# literal order, memory-mode ablations), C5 / C4 launch lists, ncu --set full of every config's
# Map and of C4's onesweep pass.
O=gpurun_out/${TAG:-ev}; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/smi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q > $O/gpu_tests.log 2>&1; echo "rc=$?" >> $O/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1
for w in C5 C4 C3 C2 C1; do
  timeout 600 python bench.py --workload $w --steps 10 --warmup 3 > $O/bench_$w.json 2> $O/bench_$w.err
done
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_reference_C5.json 2> $O/bench_reference_C5.err
timeout 900 python bench.py --scaling strong --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench_C5_strong_n1.json 2> $O/bench_C5_strong.err
timeout 600 python bench.py --no-map-combine --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench_C5_literal.json 2> $O/bench_C5_literal.err
for m in SO SI G; do for w in C5 C4 C3 C2; do
  timeout 600 python bench.py --workload $w --mode $m --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/abl_${w}_$m.json 2> $O/abl_${w}_$m.err
done; done
B="python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C5.csv $B --workload C5 > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C4.csv $B --workload C4 > /dev/null 2>&1
N="ncu --set full --clock-control none --import-source on"
for w in C5 C4 C3 C2; do
  timeout 900 $N -k regex:k_map -c 1 -o $O/r02_${w}_k_map -f $B --workload $w > $O/ncu_$w.log 2>&1
done
timeout 600 $N -k regex:k_onesweep -s 2 -c 1 -o $O/r02_C4_onesweep -f $B --workload C4 > $O/ncu_os.log 2>&1
timeout 600 $N -k regex:k_xtab_extract -c 1 -o $O/r02_C5_xtab -f $B --workload C5 > $O/ncu_xtab.log 2>&1
ls -la $O
