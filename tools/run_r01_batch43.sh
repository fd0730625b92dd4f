#!/bin/bash
# Max trainable size in host RAM (c4max) with the final GPT driver, extended autotune, settle steps.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=900
timeout 2400 python bench.py --config c4max --grow-landing --fill-gpu --late-shadow --no-cpu-baseline --no-e2e \
    > gpurun_out/c4max43.json 2> gpurun_out/c4max43.err
python - <<PY
import json
d = json.loads(open("gpurun_out/c4max43.json").read().strip().splitlines()[-1])
c = d["config"]
print("c4max", c["layers"], c["params"], c["window"], c["ring_slots"], round(d["value"], 3), "resfit", (d.get("resident_fit") or {}).get("frac_model_tflops"), "hdram", d["host_dram"]["frac"])
PY
