#!/bin/bash
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=120
timeout 600 python -m pytest tests/test_hetero_gpu.py -q -x > gpurun_out/pytest28.log 2>&1
tail -30 gpurun_out/pytest28.log
