#!/bin/bash
# A/B of the default build against variant libraries (variants/libbmr_<v>.so) and env settings,
# interleaved REPS times: AB="name:ENV=val ..." VARS="v1 v2" WL=C5 [K=pytest filter] [NCU=1]
O=gpurun_out/${TAG:-ab}; mkdir -p $O
if [ -n "$K" ]; then
  timeout 1200 python -m pytest tests -m gpu -x -q -k "$K" > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log; tail -2 $O/tests.log
fi
B="python bench.py --workload ${WL:-C5} --steps ${STEPS:-5} --warmup 3 --e2e-steps 0 --no-cpu-baseline"
for rep in ${REPS:-1 2}; do
  timeout 300 $B > $O/b_default_$rep.json 2>/dev/null
  for v in $VARS; do BMR_LIB=variants/libbmr_$v.so timeout 300 $B > $O/b_${v}_$rep.json 2>/dev/null; done
  for spec in $AB; do n=${spec%%:*}; e=${spec#*:}; env ${e//,/ } timeout 300 $B > $O/b_${n}_$rep.json 2>/dev/null; done
done
for f in $O/b_*.json; do python -c "
import json; d=json.load(open('$f')); print('$f'.split('/')[-1], d['value'], d['phases_ms']['map'], d['ms_per_step'])" 2>/dev/null || echo "$f failed"; done
if [ -n "$NCU" ]; then TAG=${TAG:-ab} NAME=${WL:-C5}_map K=k_map WL=${WL:-C5} bash tools/r03/ncu_export.sh > /dev/null 2>&1; fi
