#!/bin/bash
# The autotuned C4 with the B200 extensions of the window model: landing growth, serialised-link FP
# constraint + GPU set filling the HBM the ring leaves, late bf16 shadows.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=600
timeout 900 python -m pytest tests/test_host_store_gpu.py tests/test_autotune.py -q > gpurun_out/pytest20.log 2>&1
tail -3 gpurun_out/pytest20.log
timeout 1800 python bench.py --grow-landing --fill-gpu --late-shadow --no-cpu-baseline \
    --trace-out gpurun_out/trace_c4_tuned.json > gpurun_out/c4_tuned.json 2> gpurun_out/c4_tuned.err
tail -c 600 gpurun_out/c4_tuned.json; echo
