#!/bin/bash
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=300
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1
tail -3 gpurun_out/pytest_gpu.log
timeout 900 python bench.py --trace-out gpurun_out/trace_c4.json > gpurun_out/default.log 2>&1
tail -c 600 gpurun_out/default.log; echo
timeout 600 python bench.py --config c2 --window -1 --cpu-hard 1 --steps 10 --trace-out gpurun_out/trace_c2.json > gpurun_out/c2_auto.log 2>&1
tail -c 300 gpurun_out/c2_auto.log; echo
