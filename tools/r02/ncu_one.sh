#!/bin/bash
# ncu --set full of one kernel (regex $K) of one bench config ($WL), plus the launch list of the step
O=gpurun_out/${TAG:-ncu}; mkdir -p $O
W=${WL:-C5}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:${K:-k_map} -c 1 -o $O/${W}_${KN:-k_map} -f python bench.py --workload $W --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > $O/ncu_$W.log 2>&1
if [ -n "$LAUNCHES" ]; then
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$W.csv python bench.py --workload $W --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline > $O/launch_$W.log 2>&1
fi
