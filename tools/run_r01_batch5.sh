#!/bin/bash
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=300
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1
tail -5 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --config c2 --steps 10 > gpurun_out/c2_fa.log 2>&1
tail -c 400 gpurun_out/c2_fa.log; echo
timeout 600 python bench.py --config c2 --window -1 --cpu-hard 1 --steps 10 --no-cpu-baseline > gpurun_out/c2_fa_auto.log 2>&1
tail -c 400 gpurun_out/c2_fa_auto.log; echo
