#!/bin/bash
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=300
df -h /dev/shm > gpurun_out/shm.txt
timeout 900 python bench.py > gpurun_out/default.log 2>&1
tail -c 2500 gpurun_out/default.log; echo
timeout 600 python bench.py --config c2 --window -1 --cpu-hard 1 --steps 10 --no-cpu-baseline > gpurun_out/c2_auto85.log 2>&1
tail -c 300 gpurun_out/c2_auto85.log; echo
timeout 900 python bench.py --config c3 --steps 8 --no-e2e --no-cpu-baseline > gpurun_out/c3_auto85.log 2>&1
tail -c 300 gpurun_out/c3_auto85.log; echo
timeout 600 python bench.py --config c2 --window 48 --steps 8 --no-e2e --no-cpu-baseline --no-resident --batch 32 > gpurun_out/c2_res_b32.log 2>&1
