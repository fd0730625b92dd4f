#!/bin/bash
# Chrome trace of one profiled step of the final default C4 configuration (Fig. 4 analogue)
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=900
timeout 1500 python bench.py --no-cpu-baseline --no-resident --no-e2e --trace-out gpurun_out/trace_c4_final.json \
    > gpurun_out/c4_trace45.json 2> gpurun_out/c4_trace45.err
tail -c 200 gpurun_out/c4_trace45.json; ls -la gpurun_out/trace_c4_final.json*
