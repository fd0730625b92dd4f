#!/bin/bash
# ncu evidence for the default c4max step (run under gpurun, 1 GPU):
#  1. ncu --set full of K2 / K1 / K3 / K4 at one h=4096 layer in isolation (tools/ncu_kernels.sh)
#  2. the launch list (gpu__time_duration per launch, --clock-control none) of the default bench's
#     configuration with the window fixed to what the autotuner settles on (41 GPU layers, ring 32), so
#     the profile taken under ncu cannot change it
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
bash tools/ncu_kernels.sh > /dev/null 2>&1
python tools/ncu_iso_summary.py gpurun_out gpurun_out/r02_ncu_iso_kernels.json; cat gpurun_out/r02_ncu_iso_kernels.json | head -c 1500; echo
export SH_WAIT_TIMEOUT_S=900
timeout 2400 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/ncu_launches_c4max.csv \
    python bench.py --window 41 --ring 32 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --resident-fit-layers 0 \
    > gpurun_out/ncu_launches_c4max.log 2>&1; echo "ncu launches rc $?"
python tools/summarize_launches.py gpurun_out/ncu_launches_c4max.csv > gpurun_out/ncu_launches_c4max.txt 2>&1; head -25 gpurun_out/ncu_launches_c4max.txt
