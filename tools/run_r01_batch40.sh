#!/bin/bash
# Same-box A/B: own column-sum kernels (SH_GPT_COLSUM=1) vs cuBLAS GEMV / M=1 GEMM (0), alternating.
# (the SH_GPT_COLSUM switch and the own column-sum kernels were removed after this A/B: profiles/r01_gpt_colsum_ab.txt)
mkdir -p gpurun_out
for cs in 1 0 1 0; do
  SH_GPT_COLSUM=$cs timeout 900 python bench.py --config c4 --layers 36 --window 36 --steps 6 --no-resident --no-cpu-baseline --no-e2e \
      > gpurun_out/fit36_ab$cs.json 2> /dev/null
  SH_GPT_COLSUM=$cs timeout 900 python bench.py --config c2 --window 48 --steps 6 --no-resident --no-cpu-baseline --no-e2e \
      > gpurun_out/c2res_ab$cs.json 2> /dev/null
  python - <<PY
import json
for f in ("fit36_ab$cs", "c2res_ab$cs"):
    d = json.loads(open(f"gpurun_out/{f}.json").read().strip().splitlines()[-1])
    print(f, round(d["value"], 3), round(d["model_tflops"], 1))
PY
done
