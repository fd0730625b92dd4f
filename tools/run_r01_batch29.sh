#!/bin/bash
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=120
timeout 900 python -m pytest tests/test_hetero_gpu.py tests/test_engine_gpu.py tests/test_host_store_gpu.py -q -x > gpurun_out/pytest29.log 2>&1
tail -30 gpurun_out/pytest29.log
