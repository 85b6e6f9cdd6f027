#!/bin/bash
O=gpurun_out/${TAG:-km}; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -m gpu -x -q -k "km or KM" > $O/tests.log 2>&1; echo "rc=$?" >> $O/tests.log
WL=C3 bash tools/r02/variants.sh "$@"
