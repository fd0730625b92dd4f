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
# NEXT-2: C2 with ~8 host layers in the spill tier (pinned budget 21.5 GB), page cache kept / evicted
for ev in "" "--spill-evict"; do
  mkdir -p /tmp/sh_spill
  timeout 900 python bench.py --config c2 --steps 3 --no-resident --no-cpu-baseline --no-e2e \
      --spill-dir /tmp/sh_spill --host-pin-gb 21.5 $ev > gpurun_out/spill_c2${ev}.json 2> gpurun_out/spill_c2${ev}.err
  tail -c 400 gpurun_out/spill_c2${ev}.json; echo
done
timeout 1200 python bench.py > gpurun_out/default14.log 2>&1
tail -c 600 gpurun_out/default14.log; echo
