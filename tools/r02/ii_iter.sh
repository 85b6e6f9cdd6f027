#!/bin/bash
O=gpurun_out/${TAG:-ii}; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_multirank.py -m gpu -x -q -k "ii or II" > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
WL=C4 TAG=${TAG:-ii} bash tools/r02/env_variants.sh "fast:BMR_MAP_FAST=1" "generic:BMR_MAP_FAST=0"
