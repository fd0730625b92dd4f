#!/bin/bash
# Autotuned C4 with the B200 window-model extensions (fastest-fetch estimate for the late shadow).
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=600 SH_DEBUG_AUTOTUNE=1
timeout 1800 python bench.py --grow-landing --fill-gpu --late-shadow --no-cpu-baseline \
    --trace-out gpurun_out/trace_c4_tuned2.json > gpurun_out/c4_tuned2.json 2> gpurun_out/c4_tuned2.err
tail -c 900 gpurun_out/c4_tuned2.json; echo; grep "sh autotune" gpurun_out/c4_tuned2.err
