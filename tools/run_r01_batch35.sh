#!/bin/bash
# Which cuBLASLt epilogue helps at which width: masks 1 (qkv bias), 2 (fc bias+GELU), 4 (dGELU), 0 (none)
mkdir -p gpurun_out
for m in 0 1 2 4 7; do
  SH_GPT_LT=$m timeout 900 python bench.py --config c4 --layers 36 --window 36 --steps 6 --no-resident --no-cpu-baseline --no-e2e \
      > gpurun_out/fit36_m$m.json 2> gpurun_out/fit36_m$m.err
  SH_GPT_LT=$m timeout 900 python bench.py --config c2 --window 48 --steps 6 --no-resident --no-cpu-baseline --no-e2e \
      > gpurun_out/c2res_m$m.json 2> gpurun_out/c2res_m$m.err
  python - <<PY
import json
for f in ("fit36_m$m", "c2res_m$m"):
    d = json.loads(open(f"gpurun_out/{f}.json").read().strip().splitlines()[-1])
    print(f, round(d["value"], 3), round(d["model_tflops"], 1))
PY
done
