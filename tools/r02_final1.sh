#!/bin/bash
# Default bench with the CPU prefetch default, kernel parity tests, smoke, thread-count A/B.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc $?"
timeout 600 python -m pytest tests/test_kernels_gpu.py -x -q -m gpu > gpurun_out/pytest_kernels.log 2>&1; echo "kernels rc $?"; tail -1 gpurun_out/pytest_kernels.log
timeout 1500 python bench.py --trace-out gpurun_out/trace_default.json > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; echo "bench rc $?"
python - <<'PY'
import json
d = json.loads(open("gpurun_out/bench_default.json").read().strip().splitlines()[-1])
print(d["value"], d["e2e"]["value"], d["runs"]["samples_per_s"], d["resident_fit"]["frac_model_tflops"], d["roofline"]["frac"],
      d["host_dram"]["achieved_gbs"], d["host_dram"]["frac"], d["compute_stream"]["stall_frac"], d["config"]["window"], d["config"]["ring_slots"])
PY
bash tools/ab_c4max.sh 112 "t14||--cpu-threads 14" "t16||--cpu-threads 16"
