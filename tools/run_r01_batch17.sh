#!/bin/bash
# NEXT-2 at scale: C4 beyond host RAM (88 layers, 17.9 B params; ~15 layers in the spill tier on the
# box's virtio disk, page cache dropped after every update), then C3 and C2 refresh with the current code.
mkdir -p gpurun_out /tmp/sh_spill
export SH_WAIT_TIMEOUT_S=900
df -h /tmp > gpurun_out/df17.txt
free -g >> gpurun_out/df17.txt
timeout 2400 python bench.py --layers 88 --host-pin-gb 180 --spill-dir /tmp/sh_spill --spill-evict \
    --steps 2 --no-resident --no-e2e --no-cpu-baseline > gpurun_out/c4_spill90.json 2> gpurun_out/c4_spill90.err
tail -c 500 gpurun_out/c4_spill90.json; echo; tail -3 gpurun_out/c4_spill90.err
free -g >> gpurun_out/df17.txt
timeout 1200 python bench.py --config c3 --no-cpu-baseline > gpurun_out/c3.json 2> gpurun_out/c3.err
tail -c 300 gpurun_out/c3.json; echo
timeout 900 python bench.py --config c2 --window -1 --cpu-hard 1 --no-cpu-baseline > gpurun_out/c2_auto.json 2> gpurun_out/c2_auto.err
tail -c 300 gpurun_out/c2_auto.json; echo
