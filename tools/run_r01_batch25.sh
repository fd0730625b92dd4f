#!/bin/bash
# K2 variants, isolated microbench: register-staged (2 blocks/SM; grid 4 or 2 per SM), capped at 80
# registers (3 blocks/SM), bulk-copy pipelines (4096-element items 1 block/SM, 2048 2 blocks/SM).
mkdir -p gpurun_out
for v in "ldg 4" "ldg 2" "ldg3 3" "bulk4k 0" "bulk2k 0"; do
  set -- $v
  SH_K2_IMPL=$1 SH_K2_BPS=$2 timeout 300 python tools/bench_kernels.py > gpurun_out/kern25_$1_$2.log 2>&1
  echo "$1 bps$2"; grep K2 gpurun_out/kern25_$1_$2.log | tail -3
done
SH_K2_IMPL=bulk2k timeout 300 python -m pytest tests/test_kernels_gpu.py -q -x 2>&1 | tail -1
SH_K2_IMPL=ldg3 timeout 300 python -m pytest tests/test_kernels_gpu.py -q -x 2>&1 | tail -1
