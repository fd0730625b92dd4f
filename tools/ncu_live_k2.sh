#!/bin/bash
# ncu --set full of ONE K2 launch inside the live default bench step (a GPU-optimised h=4096 layer's
# per-layer AdamW, 201,379,840 elements, after the warm-up), beside the isolated capture of
# tools/ncu_kernels.sh.  Writes gpurun_out/ncu_live_k2.{ncu-rep,csv,log}.
mkdir -p gpurun_out
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:k2_adamw_kernel --launch-skip 300 -c 1 \
    -o gpurun_out/ncu_live_k2 -f python bench.py --steps 3 --no-e2e --resident-fit-layers 0 --no-cpu-baseline \
    > gpurun_out/ncu_live_k2.log 2>&1
ncu -i gpurun_out/ncu_live_k2.ncu-rep --page raw --csv \
    --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,launch__grid_size,launch__registers_per_thread,dram__throughput.avg.pct_of_peak_sustained_elapsed \
    > gpurun_out/ncu_live_k2.csv 2>&1
tail -3 gpurun_out/ncu_live_k2.csv
