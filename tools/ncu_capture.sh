#!/bin/bash
# ncu evidence for the hot-path kernels (run under gpurun; 1 GPU).  Writes gpurun_out/ncu_*.
set -x
mkdir -p gpurun_out
B="python bench.py --config ${CFG:-c2} --steps 1 --warmup 3 --no-resident --no-e2e --no-cpu-baseline"
# 1) every launch with its device time (cold-cache, serialised: compare shares only)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/ncu_launches.csv $B > gpurun_out/ncu_launches.log 2>&1
# 2) full sets of K2 (fused AdamW), K3 (sumsq) and K1 (cast) -- one launch each after warm-up
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k2_adamw -s 3 -c 1 \
    -o gpurun_out/ncu_k2 -f $B > gpurun_out/ncu_k2.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k3_partial -s 200 -c 1 \
    -o gpurun_out/ncu_k3 -f $B > gpurun_out/ncu_k3.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k1_cast -s 20 -c 1 \
    -o gpurun_out/ncu_k1 -f $B > gpurun_out/ncu_k1.log 2>&1
ls -la gpurun_out
