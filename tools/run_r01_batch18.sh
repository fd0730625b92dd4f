#!/bin/bash
# Fig. 14 analogue: optimisation breakdown on C2 (b16, window 4 fixed).
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=600
B="python bench.py --config c2 --steps 5 --no-resident --no-cpu-baseline --no-e2e"
for v in "base:" "threads1:--cpu-threads 1" "threads4:--cpu-threads 4" "synccpu:--sync-cpu" "alloc:--ablate-alloc"; do
  n=${v%%:*}; a=${v#*:}
  timeout 900 $B $a > gpurun_out/abl_$n.json 2> gpurun_out/abl_$n.err
  echo "$n"; tail -c 200 gpurun_out/abl_$n.json; echo
done
