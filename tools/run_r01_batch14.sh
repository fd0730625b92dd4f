#!/bin/bash
# NEXT-3 executors + K4, NEXT-2 spill tier: GPU tests, isolated ncu of K1-K4, executor and spill benches.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=300
df -h /tmp /root /dev/shm > gpurun_out/df.txt 2>&1
timeout 900 python -m pytest tests/test_kernels_gpu.py tests/test_executors_gpu.py tests/test_spill_gpu.py -q \
    > gpurun_out/pytest_new.log 2>&1
tail -3 gpurun_out/pytest_new.log
bash tools/ncu_kernels.sh > gpurun_out/ncu_kernels.log 2>&1
B="python bench.py --config c2 --steps 5 --no-resident --no-cpu-baseline --no-e2e"
for bk in "4 1" "4 2" "4 4" "16 1" "16 2"; do
  set -- $bk
  timeout 600 $B --batch $1 --executors $2 > gpurun_out/exec_b$1_k$2.json 2> gpurun_out/exec_b$1_k$2.err
  tail -c 300 gpurun_out/exec_b$1_k$2.json; echo
done
