#!/bin/bash
# Landing-ring growth at C4: coupled ring + full landing store, and decoupled ring, vs the default.
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=600
timeout 900 python -m pytest tests/test_host_store_gpu.py tests/test_autotune.py -q > gpurun_out/pytest19.log 2>&1
tail -3 gpurun_out/pytest19.log
for v in "grow_coupled:--grow-landing --no-decouple" "grow_decoupled:--grow-landing"; do
  n=${v%%:*}; a=${v#*:}
  timeout 1500 python bench.py $a --no-resident --no-cpu-baseline --no-e2e --trace-out gpurun_out/trace_c4_$n.json \
      > gpurun_out/c4_$n.json 2> gpurun_out/c4_$n.err
  echo $n; tail -c 300 gpurun_out/c4_$n.json; echo
done
# hand-picked decoupled configurations of the C4 model (81 layers): more GPU-set layers, a 16-21 slot
# ring, full landing store, bf16 shadow fetch (host RAM is free once only host layers hold blocks)
for v in "g46r21_bf16:--window 46 --ring 21 --fetch-fp32 0" "g44r16_bf16:--window 44 --ring 16 --fetch-fp32 0" \
         "g46r21_f32:--window 46 --ring 21 --fetch-fp32 1"; do
  n=${v%%:*}; a=${v#*:}
  timeout 1200 python bench.py --layers 81 --grad-ring 40 $a --no-resident --no-cpu-baseline --no-e2e \
      --trace-out gpurun_out/trace_c4_$n.json > gpurun_out/c4_$n.json 2> gpurun_out/c4_$n.err
  echo $n; tail -c 300 gpurun_out/c4_$n.json; echo
done
