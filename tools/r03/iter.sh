#!/bin/bash
# Generic iteration: pytest -m gpu -k "$K" (optional), then bench lines of "name:args" specs
# (BENCHES), then an optional ncu export (NCU="NAME K WL [ARGS]").
O=gpurun_out/${TAG:-it}; mkdir -p $O
if [ -n "$K" ]; then
  timeout 1200 python -m pytest tests -m gpu -x -q -k "$K" > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
  tail -3 $O/tests.log
fi
for rep in ${REPS:-1}; do
for spec in $BENCHES; do
  name=${spec%%:*}; a=${spec#*:}; a=${a//,/ }
  timeout 400 python bench.py --steps ${STEPS:-5} --warmup 3 --e2e-steps 0 --no-cpu-baseline $a > $O/bench_$name.json 2> $O/bench_$name.err
  python -c "
import json; d=json.load(open('$O/bench_$name.json')); print('$name', d['value'], d['ms_per_step'], d['phases_ms'], d['roofline'].get('frac'), d.get('kmeans'))" >> $O/summary.txt 2>&1 || tail -3 $O/bench_$name.err >> $O/summary.txt
done; done
if [ -n "$NCU" ]; then
  set -- $NCU
  TAG=${TAG:-it} NAME=$1 K=$2 WL=$3 ARGS="${@:4}" bash tools/r03/ncu_export.sh > /dev/null 2>&1
fi
cat $O/summary.txt
