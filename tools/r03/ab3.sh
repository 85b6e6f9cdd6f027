O=gpurun_out/ab3; mkdir -p $O
timeout 1200 python -m pytest tests -m gpu -x -q > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log; tail -3 $O/tests.log
for rep in 1 2; do for wl in C5 C4; do
  timeout 300 python bench.py --workload $wl --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/b_def_${wl}_$rep.json 2>/dev/null
  BMR_LIB=variants/libbmr_nodyn.so timeout 300 python bench.py --workload $wl --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/b_nodyn_${wl}_$rep.json 2>/dev/null
done; done
for f in $O/b_*.json; do python -c "
import json; d=json.load(open('$f')); print('$f'.split('/')[-1], d['value'], d['phases_ms']['map'], d['ms_per_step'])" 2>/dev/null || echo "$f failed"; done
