#!/bin/bash
# Full GPU suite (incl. the one-rank NCCL DP path), executors at GPU-bound small batch, spill rerun, C4 b32.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=300
timeout 1800 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu15.log 2>&1
tail -3 gpurun_out/pytest_gpu15.log
B="python bench.py --config c2 --steps 5 --no-resident --no-cpu-baseline --no-e2e"
for bk in "4 1" "4 2" "4 4" "8 1" "8 2"; do
  set -- $bk
  timeout 600 $B --window 48 --batch $1 --executors $2 > gpurun_out/exec_res_b$1_k$2.json 2> gpurun_out/exec_res_b$1_k$2.err
  tail -c 200 gpurun_out/exec_res_b$1_k$2.json; echo
done
mkdir -p /tmp/sh_spill
timeout 900 $B --spill-dir /tmp/sh_spill --host-pin-gb 21.5 > gpurun_out/spill_c2_v2.json 2> gpurun_out/spill_c2_v2.err
tail -c 300 gpurun_out/spill_c2_v2.json; echo
timeout 1500 python bench.py --batch 32 > gpurun_out/c4_b32.log 2>&1
tail -c 600 gpurun_out/c4_b32.log; echo
