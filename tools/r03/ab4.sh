# full GPU suite, then C5 / C4 benches of the default build and variant libraries (VARS)
O=gpurun_out/${TAG:-ab4}; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log; tail -3 $O/tests.log
for rep in ${REPS:-1 2}; do for wl in ${WLS:-C5}; do
  timeout 300 python bench.py --workload $wl --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/b_def_${wl}_$rep.json 2>/dev/null
  for v in $VARS; do BMR_LIB=variants/libbmr_$v.so timeout 300 python bench.py --workload $wl --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/b_${v}_${wl}_$rep.json 2>/dev/null; done
done; done
for f in $O/b_*.json; do python -c "
import json; d=json.load(open('$f')); print('$f'.split('/')[-1], d['value'], d['phases_ms']['map'], d['ms_per_step'])" 2>/dev/null || echo "$f failed"; done
