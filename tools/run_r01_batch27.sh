#!/bin/bash
# Full-size C4 parity test, engine tests (compute-stream busy), default bench with the stall report.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=600
timeout 1500 python -m pytest tests/test_fullsize_c4_gpu.py tests/test_engine_gpu.py -q > gpurun_out/pytest27.log 2>&1
tail -5 gpurun_out/pytest27.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke27.log 2>&1; tail -2 gpurun_out/smoke27.log
timeout 1800 python bench.py > gpurun_out/c4_default27.json 2> gpurun_out/c4_default27.err
tail -c 400 gpurun_out/c4_default27.json; echo
