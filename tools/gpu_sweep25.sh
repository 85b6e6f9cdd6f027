#!/bin/bash
# f-3 fused InvertedIndex flush into receive windows (virtual ranks on one GPU) + full suite
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_multirank.py -x -q > gpurun_out/xwin_tests.log 2>&1; echo "rc=$?" >> gpurun_out/xwin_tests.log
timeout 400 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "rc=$?" >> gpurun_out/gpu_tests.log
