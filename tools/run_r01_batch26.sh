#!/bin/bash
# (1) ncu launch list of the new default C4 configuration (window / ring / fetch fixed to what the
#     autotuner chose in profiles/r01_bench_default_c4_v4.json: 53 GPU-optimised layers, ring 15,
#     bf16 shadows, one landing buffer per host layer), so the K2 share can be compared with the
#     bench's live numbers; (2) c4max (max trainable size in host RAM) with the autotune extensions.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=600
B="python bench.py --layers 82 --window 53 --ring 15 --fetch-fp32 0 --grad-ring 29 --steps 1 --no-e2e --no-cpu-baseline --no-resident"
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none --csv -c 7000 \
    --log-file gpurun_out/ncu_launches_c4_v4.csv $B > gpurun_out/ncu_launches_c4_v4.log 2>&1
tail -3 gpurun_out/ncu_launches_c4_v4.log; wc -l gpurun_out/ncu_launches_c4_v4.csv
timeout 900 python bench.py --layers 82 --window 53 --ring 15 --fetch-fp32 0 --grad-ring 29 --no-e2e \
    --no-cpu-baseline --no-resident > gpurun_out/c4_fixed_v4.json 2> gpurun_out/c4_fixed_v4.err
tail -c 300 gpurun_out/c4_fixed_v4.json; echo
timeout 1800 python bench.py --config c4max --grow-landing --fill-gpu --late-shadow --no-cpu-baseline --no-e2e \
    > gpurun_out/c4max_v4.json 2> gpurun_out/c4max_v4.err
tail -c 600 gpurun_out/c4max_v4.json; echo; tail -3 gpurun_out/c4max_v4.err
