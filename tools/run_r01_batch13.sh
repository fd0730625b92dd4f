#!/bin/bash
# Re-validation after the container restore: GPU tests + default bench.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=300
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout 1800 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1
tail -3 gpurun_out/pytest_gpu.log
timeout 1200 python bench.py --trace-out gpurun_out/trace_c4.json > gpurun_out/default.log 2>&1
tail -c 1500 gpurun_out/default.log; echo
