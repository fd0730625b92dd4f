#!/bin/bash
# ncu --set full of ONE per-layer K2 launch (and one K1, one K3) inside the default C4 configuration
# (window / ring / fetch fixed to the autotuner's choice so ncu's replay cannot change them): DRAM
# traffic per launch in the live setting, beside the isolated captures.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=900
B="python bench.py --layers 82 --window 53 --ring 16 --fetch-fp32 0 --grad-ring 29 --steps 1 --no-e2e --no-cpu-baseline --no-resident"
for k in k2_adamw k1_cast k3_sumsq; do
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:$k -s 60 -c 1 \
      -o gpurun_out/ncu_live_$k -f $B > gpurun_out/ncu_live_$k.log 2>&1
  ncu -i gpurun_out/ncu_live_$k.ncu-rep --page raw --csv \
      --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,launch__grid_size,launch__registers_per_thread,dram__throughput.avg.pct_of_peak_sustained_elapsed \
      > gpurun_out/ncu_live_$k.csv 2>&1
  tail -2 gpurun_out/ncu_live_$k.csv
done
