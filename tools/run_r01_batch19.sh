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
