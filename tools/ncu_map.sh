#!/bin/bash
B="python bench.py --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_map -s 1 -c 1 -o gpurun_out/prof3_C5_k_map -f $B --workload C5 --units 1024 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_onesweep -s 3 -c 1 -o gpurun_out/prof3_C5_k_onesweep -f $B --workload C5 --units 1024 > /dev/null 2>&1
for i in 1 2; do python bench.py --workload C4 --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline | python -c "import json,sys;d=json.loads(sys.stdin.read());print(d['value'],d['ms_per_step'],d['phases_ms'],d['wall_s_timed'])"; done
