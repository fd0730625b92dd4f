#!/bin/bash
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=300
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1
tail -5 gpurun_out/pytest_gpu.log
for cfg in "2 4" "4 4" "2 8" "4 2"; do set -- $cfg
  SH_K2_U=$1 SH_K2_BPS=$2 timeout 300 python tools/bench_kernels.py > gpurun_out/kern_u$1_b$2.log 2>&1
  echo "U=$1 BPS=$2"; grep K2 gpurun_out/kern_u$1_b$2.log
done
grep -E "K1|K3" gpurun_out/kern_u2_b4.log
timeout 900 python bench.py --config c3 --layers 36 --window 36 --steps 6 --no-e2e --no-cpu-baseline --no-resident > gpurun_out/c3_resfit.log 2>&1
tail -c 400 gpurun_out/c3_resfit.log
