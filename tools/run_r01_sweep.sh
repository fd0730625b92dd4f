#!/bin/bash
# Round-1 measurement batch (run under gpurun): GPU tests, C2 window sweep (Fig. 9
# analogue), C2 batch 32, C3 10B.  Outputs gpurun_out/*.json|log.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=300
timeout 600 python -m pytest tests -q -m gpu -x > gpurun_out/pytest_gpu.log 2>&1
tail -3 gpurun_out/pytest_gpu.log
for w in 1 2 8 16; do
  timeout 400 python bench.py --config c2 --window $w --steps 8 --no-resident --no-e2e --no-cpu-baseline \
     > gpurun_out/sweep_c2_w$w.log 2>&1; tail -c 400 gpurun_out/sweep_c2_w$w.log | head -c 200; echo
done
timeout 600 python bench.py --config c2 --batch 32 --window 4 --steps 8 --no-e2e --no-cpu-baseline \
   > gpurun_out/c2_b32.log 2>&1
timeout 1200 python bench.py --config c3 --window 4 --grad-ring 8 --steps 5 --no-e2e --no-cpu-baseline \
   > gpurun_out/c3_b16.log 2>&1
free -g > gpurun_out/free.txt
tail -2 gpurun_out/c3_b16.log | head -c 600
