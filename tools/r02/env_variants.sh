#!/bin/bash
# bench one workload under several environment settings: env_variants.sh "NAME=VAR=val ..." ...
O=gpurun_out/${TAG:-envv}; mkdir -p $O
W=${WL:-C5}
for spec in "$@"; do
  name=${spec%%:*}; envs=${spec#*:}
  env $envs timeout 300 python bench.py --workload $W --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench_$name.json 2> $O/bench_$name.err
  python -c "
import json; d=json.load(open('$O/bench_$name.json')); print('$name', d['value'], d['ms_per_step'], d['phases_ms'])"
done
