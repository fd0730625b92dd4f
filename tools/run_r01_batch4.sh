#!/bin/bash
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=300
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1
tail -5 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --config c2 --steps 10 --trace-out gpurun_out/trace_c2.json > gpurun_out/c2.log 2>&1
tail -c 300 gpurun_out/c2.log; echo
export SH_HOST_MARGIN_GB=6
timeout 1500 python bench.py --config c4 --steps 5 --no-e2e --no-cpu-baseline --trace-out gpurun_out/trace_c4.json > gpurun_out/c4_auto.log 2>&1
tail -c 1500 gpurun_out/c4_auto.log; echo
timeout 1200 python bench.py --config c3 --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/c3_auto.log 2>&1
tail -c 600 gpurun_out/c3_auto.log
