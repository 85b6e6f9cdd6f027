#!/bin/bash
# WordCount Map iteration: WC parity tests, C5 bench (fast path vs previous path), ncu of k_map<1>.
O=gpurun_out/${TAG:-wc}; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -m gpu -x -q -k "wc or WC" > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
timeout 300 python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench_fast.json 2> $O/bench_fast.err
BMR_WC_FAST=0 timeout 300 python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench_old.json 2> $O/bench_old.err
if [ -n "$NCU" ]; then
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_map -c 1 -o $O/C5_k_map -f python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > $O/ncu.log 2>&1
fi
tail -3 $O/tests.log
