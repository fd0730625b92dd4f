#!/bin/bash
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=300
timeout 1200 python -m pytest tests/test_engine_gpu.py -q -k "ring_smaller or autotune or delay" > gpurun_out/pytest_ring.log 2>&1
tail -3 gpurun_out/pytest_ring.log
timeout 900 python bench.py --trace-out gpurun_out/trace_c4.json > gpurun_out/default.log 2>&1
tail -c 1800 gpurun_out/default.log; echo
timeout 900 python bench.py --config c3 --steps 8 --no-e2e --no-cpu-baseline > gpurun_out/c3_dec.log 2>&1
tail -c 500 gpurun_out/c3_dec.log; echo
timeout 600 python bench.py --config c2 --window -1 --cpu-hard 1 --steps 10 --no-cpu-baseline > gpurun_out/c2_dec.log 2>&1
tail -c 300 gpurun_out/c2_dec.log; echo
