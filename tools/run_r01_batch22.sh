#!/bin/bash
# Same box, back to back, twice: autotuned (extensions on) vs the hand-picked decoupled C4 configuration.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=600 SH_DEBUG_AUTOTUNE=1
for rep in 1 2; do
  timeout 1200 python bench.py --grow-landing --fill-gpu --late-shadow --no-cpu-baseline --no-resident --no-e2e \
      > gpurun_out/c4_auto_r$rep.json 2> gpurun_out/c4_auto_r$rep.err
  echo auto$rep; tail -c 200 gpurun_out/c4_auto_r$rep.json; echo; grep "sh autotune" gpurun_out/c4_auto_r$rep.err
  timeout 1200 python bench.py --layers 82 --grad-ring 40 --window 46 --ring 21 --fetch-fp32 0 --no-cpu-baseline \
      --no-resident --no-e2e > gpurun_out/c4_fixed_r$rep.json 2> gpurun_out/c4_fixed_r$rep.err
  echo fixed$rep; tail -c 200 gpurun_out/c4_fixed_r$rep.json; echo
done
