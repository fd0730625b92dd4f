#!/bin/bash
# GPT driver: MUFU tanh in the bf16 GELU kernels, unrolled LN loops.  Oracle parity of the bf16 /
# fp32 paths, then C2 and the default C4 bench.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=600
timeout 1200 python -m pytest tests/test_engine_gpu.py tests/test_ragged_gpu.py tests/test_executors_gpu.py tests/test_fullsize_gpu.py -q -x > gpurun_out/pytest30.log 2>&1
tail -3 gpurun_out/pytest30.log
timeout 900 python bench.py --config c2 --no-cpu-baseline --no-e2e > gpurun_out/c2_30.json 2> gpurun_out/c2_30.err
tail -c 300 gpurun_out/c2_30.json; echo
timeout 1800 python bench.py > gpurun_out/c4_default30.json 2> gpurun_out/c4_default30.err
tail -c 300 gpurun_out/c4_default30.json; echo
