#!/bin/bash
# GPT driver bf16 path on cuBLASLt fused epilogues (bias, bias+GELU with aux, dGELU): oracle parity +
# bitwise windows, then A/B against the SIMT passes (SH_GPT_LT=0) on the same box.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=600
timeout 1500 python -m pytest tests/test_engine_gpu.py tests/test_ragged_gpu.py tests/test_executors_gpu.py tests/test_fullsize_gpu.py tests/test_kernels_gpu.py -q -x > gpurun_out/pytest34.log 2>&1
tail -3 gpurun_out/pytest34.log
for lt in 1 0; do
  SH_GPT_LT=$lt timeout 900 python bench.py --config c4 --layers 36 --window 36 --no-resident --no-cpu-baseline --no-e2e \
      > gpurun_out/fit36_lt$lt.json 2> gpurun_out/fit36_lt$lt.err
  SH_GPT_LT=$lt timeout 900 python bench.py --config c2 --window 48 --no-resident --no-cpu-baseline --no-e2e \
      > gpurun_out/c2res_lt$lt.json 2> gpurun_out/c2res_lt$lt.err
  python - <<PY
import json
for f in ("fit36_lt$lt", "c2res_lt$lt"):
    d = json.loads(open(f"gpurun_out/{f}.json").read().strip().splitlines()[-1])
    print(f, round(d["value"], 3), round(d["model_tflops"], 1), d["gpu_launches"])
PY
done
