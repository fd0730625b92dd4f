#!/bin/bash
# Final state of the session: full GPU suite, smoke, default bench, C2 default bench.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=600
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/pytest38.log 2>&1
tail -3 gpurun_out/pytest38.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke38.log 2>&1; tail -1 gpurun_out/smoke38.log
timeout 1800 python bench.py > gpurun_out/c4_default38.json 2> gpurun_out/c4_default38.err
tail -c 300 gpurun_out/c4_default38.json; echo
timeout 900 python bench.py --config c2 > gpurun_out/c2_default38.json 2> gpurun_out/c2_default38.err
tail -c 300 gpurun_out/c2_default38.json; echo
