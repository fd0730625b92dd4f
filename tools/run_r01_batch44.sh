#!/bin/bash
# c4max (112 x 4096): decoupled ring with a partial landing ring vs the autotuner's coupled window 38.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=900
for v in "49 16 16" "46 21 24"; do
  set -- $v
  timeout 1500 python bench.py --config c4max --layers 112 --window $1 --ring $2 --grad-ring $3 --no-cpu-baseline --no-e2e --no-resident \
      > gpurun_out/c4max_w$1_r$2_d$3.json 2> gpurun_out/c4max_w$1_r$2_d$3.err
  python - <<PY
import json
d = json.loads(open("gpurun_out/c4max_w$1_r$2_d$3.json").read().strip().splitlines()[-1])
print("w$1 r$2 d$3", round(d["value"], 3), "stall", round(d["compute_stream"]["stall_frac"], 3), "hdram", round(d["host_dram"]["frac"], 3), "wait", round(d["cpu_adam"]["prefetch_wait_ms_per_step"], 1))
PY
done
