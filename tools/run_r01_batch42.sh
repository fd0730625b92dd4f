#!/bin/bash
# C2 with the extended autotuner (eq. 3 term, decoupled ring, GPU set filling HBM)
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=300
timeout 900 python bench.py --config c2 --window -1 --cpu-hard 1 --grow-landing --fill-gpu --steps 8 --no-e2e --no-cpu-baseline \
   > gpurun_out/c2_tuned42.json 2> gpurun_out/c2_tuned42.err
python - <<PY
import json
d = json.loads(open("gpurun_out/c2_tuned42.json").read().strip().splitlines()[-1])
c = d["config"]
print("c2 tuned", c["window"], c["ring_slots"], round(d["value"], 2), "resident", d.get("resident"), "stall", d["compute_stream"]["stall_frac"])
PY
