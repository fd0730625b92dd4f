#!/bin/bash
# A/B of the c4max step (pinned depth) over CPU-Adam thread counts and the offload order.
# usage (on the GPU box): bash tools/ab_c4max.sh "12 14 16" "lowest fifo" [layers]
L=${3:-106}
for T in $1; do for O in $2; do
  SH_D2H_ORDER=$O timeout 900 python bench.py --config c4max --layers $L --cpu-threads $T --no-cpu-baseline --no-e2e \
    --resident-fit-layers 0 --steps 6 > gpurun_out/ab_T${T}_${O}.json 2> gpurun_out/ab_T${T}_${O}.err
  python - "$T" "$O" <<'PY'
import json, sys
d = json.loads(open(f"gpurun_out/ab_T{sys.argv[1]}_{sys.argv[2]}.json").read().strip().splitlines()[-1])
print(sys.argv[1], sys.argv[2], round(d["value"], 3), round(d["host_dram"]["achieved_gbs"], 1),
      round(d["compute_stream"]["stall_frac"], 3), round(d["cpu_adam"]["dram_gbs"], 1), flush=True)
PY
done; done
