#!/bin/bash
# ncu launch list of the all-resident h4096 model (GPT-driver kernel times after the Lt epilogues)
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -c 2500 \
    --log-file gpurun_out/ncu_fit36.csv python bench.py --config c4 --layers 36 --window 36 --steps 1 --no-resident --no-cpu-baseline --no-e2e \
    > gpurun_out/ncu_fit36.log 2>&1
tail -2 gpurun_out/ncu_fit36.log
