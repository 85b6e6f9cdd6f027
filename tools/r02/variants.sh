#!/bin/bash
# bench C5 with each variant library given as arguments (variants/libbmr_<name>.so) and the default build
O=gpurun_out/${TAG:-var}; mkdir -p $O
W=${WL:-C5}
timeout 300 python bench.py --workload $W --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench_default.json 2> $O/bench_default.err
for v in "$@"; do
  BMR_LIB=variants/libbmr_$v.so timeout 300 python bench.py --workload $W --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench_$v.json 2> $O/bench_$v.err
done
for f in $O/bench_*.json; do python -c "
import json,sys; d=json.load(open('$f')); print('$f', d['value'], d['ms_per_step'], d['phases_ms'])"; done
