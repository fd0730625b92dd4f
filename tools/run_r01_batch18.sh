#!/bin/bash
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=600
timeout 900 python -m pytest tests/test_host_store_gpu.py tests/test_dp_path_gpu.py tests/test_executors_gpu.py \
    tests/test_spill_gpu.py tests/test_engine_gpu.py -q > gpurun_out/pytest18.log 2>&1
tail -3 gpurun_out/pytest18.log
timeout 2000 python bench.py --config c4max --no-cpu-baseline > gpurun_out/c4max.json 2> gpurun_out/c4max.err
tail -c 400 gpurun_out/c4max.json; echo
timeout 900 python bench.py --config c2 --window -1 --cpu-hard 1 --no-cpu-baseline > gpurun_out/c2_auto18.json 2> gpurun_out/c2_auto18.err
tail -c 300 gpurun_out/c2_auto18.json; echo
# Fig. 14 analogue: optimisation breakdown on C2 (b16, window 4 fixed).
B="python bench.py --config c2 --steps 5 --no-resident --no-cpu-baseline --no-e2e"
for v in "base:" "threads1:--cpu-threads 1" "threads4:--cpu-threads 4" "synccpu:--sync-cpu" "alloc:--ablate-alloc"; do
  n=${v%%:*}; a=${v#*:}
  timeout 900 $B $a > gpurun_out/abl_$n.json 2> gpurun_out/abl_$n.err
  echo "$n"; tail -c 200 gpurun_out/abl_$n.json; echo
done
# NEXT-4 / Fig. 13 analogue: FP-only streaming inference (KD teacher) of the C2 model and of the C4 model
timeout 900 python bench.py --config c2 --fp-only --steps 10 --no-resident --no-cpu-baseline > gpurun_out/fponly_c2.json 2> gpurun_out/fponly_c2.err
tail -c 300 gpurun_out/fponly_c2.json; echo
timeout 1500 python bench.py --fp-only --window 40 --steps 5 --no-resident --no-cpu-baseline > gpurun_out/fponly_c4.json 2> gpurun_out/fponly_c4.err
tail -c 300 gpurun_out/fponly_c4.json; echo
