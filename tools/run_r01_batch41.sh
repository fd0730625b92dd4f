#!/bin/bash
# C2 (configs[1]) window sweep 1..8 + all-resident + autotuned, final GPT driver (Fig. 9 analogue).
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=300
for w in 1 2 3 4 6 8 48 -1; do
  timeout 600 python bench.py --config c2 --window $w --steps 8 --no-resident --no-e2e --no-cpu-baseline \
     > gpurun_out/sweep41_c2_w$w.json 2> gpurun_out/sweep41_c2_w$w.err
  python - <<PY
import json
d = json.loads(open("gpurun_out/sweep41_c2_w$w.json").read().strip().splitlines()[-1])
c = d["config"]
print("w=$w", "window", c["window"], "ring", c["ring_slots"], round(d["value"], 2), "samples/s",
      "stall", round(d["compute_stream"]["stall_frac"] or 0, 3), "h2d", d["host_link"]["h2d_frac"], "d2h", d["host_link"]["d2h_frac"])
PY
done
