#!/bin/bash
# ncu launch list of the default bench command (C4, window fixed to the autotuned 40 so the warm-up
# profile taken under ncu cannot change it), plus full-set captures of K1/K3 at C4 shapes.
# K2 full-set replay at C4 would need ncu to back up ~100 GB of written state: captured at C2 instead
# (same kernel; profiles/r01_ncu_summary.md).
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=600
B="python bench.py --window 40 --steps 1 --no-e2e --no-cpu-baseline"
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/ncu_launches_c4.csv $B > gpurun_out/ncu_launches_c4.log 2>&1
tail -3 gpurun_out/ncu_launches_c4.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k1_cast -s 100 -c 1 \
    -o gpurun_out/ncu_k1_c4 -f $B > gpurun_out/ncu_k1_c4.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k3_sumsq -s 150 -c 1 \
    -o gpurun_out/ncu_k3_c4 -f $B > gpurun_out/ncu_k3_c4.log 2>&1
ls -la gpurun_out | tail
