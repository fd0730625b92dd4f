#!/bin/bash
# Host-DRAM contention between the CPU Adam and the copy engines: default C4 with 16 vs 12 CPU Adam
# threads, twice each on the same box (run-to-run variance).
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=600
for rep in 1 2; do
  for th in 16 12; do
    timeout 900 python bench.py --cpu-threads $th --no-resident --no-cpu-baseline --no-e2e \
        > gpurun_out/c4_th${th}_r$rep.json 2> gpurun_out/c4_th${th}_r$rep.err
    python - <<PY
import json
d = json.loads(open("gpurun_out/c4_th${th}_r$rep.json").read().strip().splitlines()[-1])
print("th${th} r$rep", round(d["value"], 3), d["config"]["window"], d["config"]["ring_slots"],
      round(d["host_link"]["h2d_frac"], 3), round(d["host_link"]["d2h_frac"], 3),
      round(d["cpu_adam"]["prefetch_wait_ms_per_step"], 1), d["compute_stream"]["stall_ms"])
PY
  done
done
