#!/bin/bash
# bench.py contract checks: N=1 default line, reference arm, --gpus 2 relaunch (shared GPU plumbing
# test), strong scaling C5 at N=1 (64 GiB in 8 GiB batches), C1 (us), C3 (fp32 roofline)
O=gpurun_out/${TAG:-bc}; mkdir -p $O
timeout 400 python bench.py --steps 5 --warmup 3 > $O/bench_C5.json 2> $O/bench_C5.err
timeout 300 python bench.py --impl reference --steps 2 --warmup 3 > $O/bench_ref.json 2> $O/bench_ref.err
BMR_SHARE_GPU=1 timeout 400 python bench.py --gpus 2 --steps 3 --warmup 3 --units 1024 --e2e-steps 1 > $O/bench_C5_g2.json 2> $O/bench_C5_g2.err
BMR_SHARE_GPU=1 timeout 400 python bench.py --gpus 2 --workload C4 --steps 3 --warmup 3 --units 1024 --e2e-steps 0 > $O/bench_C4_g2.json 2> $O/bench_C4_g2.err
BMR_SHARE_GPU=1 timeout 400 python bench.py --gpus 2 --workload C3 --steps 3 --warmup 3 --units 4194304 --e2e-steps 0 > $O/bench_C3_g2.json 2> $O/bench_C3_g2.err
timeout 900 python bench.py --scaling strong --steps 3 --warmup 3 --e2e-steps 0 --no-cpu-baseline > $O/bench_C5_strong1.json 2> $O/bench_C5_strong1.err
timeout 300 python bench.py --workload C1 --steps 20 --warmup 5 > $O/bench_C1.json 2> $O/bench_C1.err
timeout 300 python bench.py --workload C3 --steps 5 --warmup 3 > $O/bench_C3.json 2> $O/bench_C3.err
for f in $O/*.json; do echo "== $f"; head -c 600 $f; echo; done
