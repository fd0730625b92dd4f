#!/bin/bash
# K3 of host layers on its own stream (the D2H copy no longer queues behind it): engine / DP-path /
# shared-store / clip / full-size tests, then the default bench.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=600
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/pytest46.log 2>&1
tail -3 gpurun_out/pytest46.log
timeout 1800 python bench.py --no-cpu-baseline > gpurun_out/c4_default46.json 2> gpurun_out/c4_default46.err
python - <<PY
import json
d = json.loads(open("gpurun_out/c4_default46.json").read().strip().splitlines()[-1])
c = d["config"]
print("c4", c["layers"], c["window"], c["ring_slots"], round(d["value"], 3), "e2e", round(d["e2e"]["value"], 3),
      "resfit", d["resident_fit"]["frac_model_tflops"], "d2h", d["host_link"]["d2h_frac"], "h2d", d["host_link"]["h2d_frac"],
      "k3", d["roofline"]["k3_frac"], "stall", d["compute_stream"]["stall_frac"])
PY
