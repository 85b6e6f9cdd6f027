O=gpurun_out/ab16; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -x -q -k "wc_ or WC or smoke or table" > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log; tail -2 $O/tests.log
for rep in 1 2; do
 timeout 300 python bench.py --workload C5 --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/c5_def_$rep.json 2>/dev/null
 BMR_LIB=variants/libbmr_prev.so timeout 300 python bench.py --workload C5 --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/c5_prev_$rep.json 2>/dev/null
 timeout 300 python bench.py --workload C1 --steps 20 --warmup 5 --e2e-steps 0 --no-cpu-baseline > $O/c1_def_$rep.json 2>/dev/null
 BMR_MAP_WAIT=0 timeout 300 python bench.py --workload C1 --steps 20 --warmup 5 --e2e-steps 0 --no-cpu-baseline > $O/c1_w0_$rep.json 2>/dev/null
done
for f in $O/*.json; do python -c "
import json; d=json.load(open('$f')); print('$f'.split('/')[-1], d['value'], d['ms_per_step'], d['phases_ms'])"; done
