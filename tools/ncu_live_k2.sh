#!/bin/bash
# ncu --set full of ONE K2 launch inside a live training step (a GPU-optimised layer's per-layer AdamW,
# after the warm-up), beside the isolated h=4096 capture of tools/ncu_kernels.sh.  C2 (1.5 B): at c4max
# the HBM and the host RAM are full, and ncu's save/restore of the kernel's in-place p / m / v for the
# replay passes got the process killed.  Writes gpurun_out/ncu_live_k2.{ncu-rep,csv,log}.
mkdir -p gpurun_out
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:k2_adamw_kernel --launch-skip 20 -c 1 \
    -o gpurun_out/ncu_live_k2 -f python bench.py --config c2 --steps 3 --no-e2e --no-resident --no-cpu-baseline \
    > gpurun_out/ncu_live_k2.log 2>&1
ncu -i gpurun_out/ncu_live_k2.ncu-rep --page raw --csv \
    --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,launch__grid_size,launch__registers_per_thread,dram__throughput.avg.pct_of_peak_sustained_elapsed \
    > gpurun_out/ncu_live_k2.csv 2>&1
tail -3 gpurun_out/ncu_live_k2.csv
