#!/bin/bash
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=300
for r in 8 12; do
  timeout 900 python bench.py --grad-ring $r --steps 6 --no-e2e --no-cpu-baseline > gpurun_out/c4_ring$r.log 2>&1
  echo "ring $r"; tail -c 300 gpurun_out/c4_ring$r.log; echo
done
timeout 900 python bench.py --config c2 --precision fp32 --window 4 --steps 5 --no-e2e --no-cpu-baseline > gpurun_out/c2_fp32_w4.log 2>&1
tail -c 400 gpurun_out/c2_fp32_w4.log; echo
