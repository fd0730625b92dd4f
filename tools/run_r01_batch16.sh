#!/bin/bash
# Re-run the tests touched since batch15, compute-sanitizer over the new paths, isolated ncu of K1-K4,
# and the ncu launch list of the default bench command.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=300
timeout 1200 python -m pytest tests/test_fullsize_gpu.py tests/test_kernels_gpu.py tests/test_executors_gpu.py \
    tests/test_dp_path_gpu.py -q > gpurun_out/pytest16.log 2>&1
tail -3 gpurun_out/pytest16.log
bash tools/ncu_kernels.sh > gpurun_out/ncu_kernels.log 2>&1
bash tools/sanitize.sh > gpurun_out/sanitize.log 2>&1
cat gpurun_out/sanitize.log
export SH_WAIT_TIMEOUT_S=600
timeout 1800 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/ncu_launches_c4.csv python bench.py --window 40 --steps 1 --no-e2e --no-cpu-baseline \
    --no-resident > gpurun_out/ncu_launches_c4.log 2>&1
tail -2 gpurun_out/ncu_launches_c4.log | cut -c1-300
