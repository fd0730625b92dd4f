#!/bin/bash
# ncu --set full of K2 / K1 / K3 / K4 at one h=4096 layer (201,379,840 elements), isolated through the
# C-ABI op entry points (tools/kernel_once.py).  Run under gpurun (1 GPU).  Writes gpurun_out/ncu_iso_*.
mkdir -p gpurun_out
for k in k2_adamw k1_cast k3_sumsq k4_exec_reduce; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$k -s 1 -c 1 \
      -o gpurun_out/ncu_iso_$k -f python tools/kernel_once.py > gpurun_out/ncu_iso_$k.log 2>&1
  ncu -i gpurun_out/ncu_iso_$k.ncu-rep --page raw --csv \
      --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,launch__grid_size,launch__registers_per_thread \
      > gpurun_out/ncu_iso_$k.csv 2>&1
done
ls -la gpurun_out | tail -20
