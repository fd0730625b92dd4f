#!/bin/bash
# Register-cached LN kernels: parity (GPT-driver paths at h 72 / 256 / 1600), then A/B vs the
# two-pass kernels (SH_GPT_LN_REG=0) on the same box.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=600
timeout 1500 python -m pytest tests/test_engine_gpu.py tests/test_ragged_gpu.py tests/test_executors_gpu.py tests/test_fullsize_gpu.py -q -x > gpurun_out/pytest37.log 2>&1
tail -3 gpurun_out/pytest37.log
for reg in 1 0 1; do
  SH_GPT_LN_REG=$reg timeout 900 python bench.py --config c4 --layers 36 --window 36 --steps 6 --no-resident --no-cpu-baseline --no-e2e \
      > gpurun_out/fit36_ln$reg.json 2> gpurun_out/fit36_ln$reg.err
  SH_GPT_LN_REG=$reg timeout 900 python bench.py --config c2 --window 48 --steps 6 --no-resident --no-cpu-baseline --no-e2e \
      > gpurun_out/c2res_ln$reg.json 2> gpurun_out/c2res_ln$reg.err
  python - <<PY
import json
for f in ("fit36_ln$reg", "c2res_ln$reg"):
    d = json.loads(open(f"gpurun_out/{f}.json").read().strip().splitlines()[-1])
    print(f, round(d["value"], 3), round(d["model_tflops"], 1))
PY
done
