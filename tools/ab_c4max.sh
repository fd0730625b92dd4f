#!/bin/bash
# A/B of the c4max step (pinned depth): bash tools/ab_c4max.sh LAYERS "NAME|ENV|ARGS" ...
#   e.g. bash tools/ab_c4max.sh 106 "split_T14||--cpu-threads 14" "fetch32_T14||--cpu-threads 14 --fetch-fp32 1"
L=$1; shift
for spec in "$@"; do
  IFS='|' read -r NAME ENVS ARGS <<< "$spec"
  env $ENVS timeout 900 python bench.py --config c4max --layers $L --no-cpu-baseline --no-e2e --resident-fit-layers 0 \
    --steps 6 $ARGS > gpurun_out/ab_$NAME.json 2> gpurun_out/ab_$NAME.err
  python - "$NAME" <<'PY'
import json, sys
try:
    d = json.loads(open(f"gpurun_out/ab_{sys.argv[1]}.json").read().strip().splitlines()[-1])
    print(sys.argv[1], round(d["value"], 3), "dram", round(d["host_dram"]["achieved_gbs"], 1),
          "B/param", round(d["host_dram"]["bytes_per_host_param"], 1), "stall", round(d["compute_stream"]["stall_frac"], 3),
          "h2d", round(d["host_link"]["h2d_gbs_per_transfer"] or 0, 1), "d2h", round(d["host_link"]["d2h_gbs_per_transfer"] or 0, 1),
          "win", d["config"]["window"], flush=True)
except Exception as e:
    print(sys.argv[1], "FAILED", e, flush=True)
PY
done
