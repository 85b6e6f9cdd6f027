#!/bin/bash
# ncu --set full (with source) of one kernel of one bench workload; the report stays on the box
# (too large to merge back), its raw / source / details pages come back as CSV.
# usage: NAME=C5_map K=k_map WL=C5 [S=skip] tools/r03/ncu_export.sh
O=gpurun_out/${TAG:-ncu}; mkdir -p $O
R=/tmp/$NAME.ncu-rep
timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s ${S:-0} -c 1 -o ${R%.ncu-rep} -f \
  python bench.py --steps 1 --warmup 0 --e2e-steps 0 --no-cpu-baseline --workload ${WL:-C5} ${ARGS} > $O/ncu_$NAME.log 2>&1
ncu -i $R --page raw --csv > $O/${NAME}_raw.csv 2>&1
ncu -i $R --page source --csv --print-source sass | gzip > $O/${NAME}_sass.csv.gz
ncu -i $R --page source --csv --print-source cuda,sass | gzip > $O/${NAME}_src.csv.gz
ls -la $O
