#!/bin/bash
# Re-entry check of HEAD on a fresh box: full GPU suite, the new default bench (C4 with the tuned
# autotune extensions on by default), C3 with the same defaults, ncu launch list of the default C4.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=600
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest23.log 2>&1
tail -3 gpurun_out/pytest23.log
timeout 1800 python bench.py > gpurun_out/c4_default23.json 2> gpurun_out/c4_default23.err
tail -c 400 gpurun_out/c4_default23.json; echo
timeout 1200 python bench.py --config c3 --no-cpu-baseline > gpurun_out/c3_default23.json 2> gpurun_out/c3_default23.err
tail -c 300 gpurun_out/c3_default23.json; echo
