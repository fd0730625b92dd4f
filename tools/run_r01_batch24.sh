#!/bin/bash
# K2 bulk-copy pipeline variant vs the register-staged kernel (isolated microbench, parity under the
# bulk variant), NUMA placement GPU test.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=300
timeout 600 python -m pytest tests/test_host_store_gpu.py -q -k numa > gpurun_out/pytest24_numa.log 2>&1
tail -2 gpurun_out/pytest24_numa.log
SH_K2_IMPL=bulk timeout 600 python -m pytest tests/test_kernels_gpu.py tests/test_engine_gpu.py -q -x > gpurun_out/pytest24_bulk.log 2>&1
tail -2 gpurun_out/pytest24_bulk.log
for impl in ldg bulk; do
  SH_K2_IMPL=$impl timeout 300 python tools/bench_kernels.py > gpurun_out/kern24_$impl.log 2>&1
  echo $impl; grep K2 gpurun_out/kern24_$impl.log
done
