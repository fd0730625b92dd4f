#!/bin/bash
# Final default bench (K3 stream, 4 settle steps), full contract line.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=600
timeout 1800 python bench.py > gpurun_out/c4_default47.json 2> gpurun_out/c4_default47.err
python - <<PY
import json
d = json.loads(open("gpurun_out/c4_default47.json").read().strip().splitlines()[-1])
c = d["config"]
print("c4", c["layers"], c["window"], c["ring_slots"], c["settle_steps"], round(d["value"], 3), "e2e", round(d["e2e"]["value"], 3),
      "resfit", d["resident_fit"]["frac_model_tflops"], "d2h", d["host_link"]["d2h_frac"], "h2d", d["host_link"]["h2d_frac"],
      "k2", d["roofline"]["frac"], "k3", d["roofline"]["k3_frac"], "stall", d["compute_stream"]["stall_frac"])
PY
