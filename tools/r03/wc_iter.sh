#!/bin/bash
# WordCount Map iteration: WC parity tests, C5 bench under env variants (VARS="name:ENV=v ..."),
# optional ncu export of k_map (NCU=1).
O=gpurun_out/${TAG:-wc}; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -m gpu -x -q -k "wc or WC or smoke" > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
for rep in ${REPS:-1}; do for spec in ${VARS:-def:X=1}; do
  name=${spec%%:*}; envs=${spec#*:}
  env $envs timeout 300 python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline ${ARGS} > $O/bench_$name.json 2> $O/bench_$name.err
  python -c "
import json; d=json.load(open('$O/bench_$name.json')); print('$name', d['value'], d['ms_per_step'], d['phases_ms'])" >> $O/summary.txt 2>&1
done; done
if [ -n "$NCU" ]; then TAG=${TAG:-wc} NAME=C5_map K=k_map WL=C5 bash tools/r03/ncu_export.sh > /dev/null 2>&1; fi
tail -3 $O/tests.log; cat $O/summary.txt
