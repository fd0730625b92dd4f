#!/bin/bash
# GPU tests after the K3/NT/fetch-fp32/host-block changes; ncu launch list (C2) + K3 full set;
# C4 max-trainable-size run.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=300
timeout 900 python -m pytest tests -q -m gpu -x > gpurun_out/pytest_gpu.log 2>&1
tail -3 gpurun_out/pytest_gpu.log
B="python bench.py --config c2 --steps 1 --warmup 3 --no-resident --no-e2e --no-cpu-baseline"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/ncu_launches2.csv $B > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k3_sumsq -s 100 -c 1 \
    -o gpurun_out/ncu_k3 -f $B > gpurun_out/ncu_k3.log 2>&1
export SH_HOST_MARGIN_GB=6
timeout 1500 python bench.py --config c4 --steps 4 --no-e2e --no-cpu-baseline > gpurun_out/c4.log 2>&1
tail -c 1500 gpurun_out/c4.log
free -g
