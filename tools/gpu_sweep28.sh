#!/bin/bash
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_ipc.py -x -q > gpurun_out/ipc_tests.log 2>&1; echo "rc=$?" >> gpurun_out/ipc_tests.log
timeout 400 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "rc=$?" >> gpurun_out/gpu_tests.log
