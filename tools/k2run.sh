#!/bin/bash
# K2 schedule / build variants beside the live step's concurrent traffic (tools/k2_contention.py) + the
# kernel and engine parity tests under the default schedule.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
rm -f gpurun_out/k2_contention.jsonl
for v in "SH_K2_SCHED=static" "SH_K2_SCHED=dyn" "SH_K2_SCHED=dyn SH_K2_IMPL=ldg3" "SH_K2_SCHED=static SH_K2_IMPL=ldg3"; do
  env $v timeout 300 python tools/k2_contention.py "$v" >> gpurun_out/k2_contention.jsonl 2>> gpurun_out/k2_contention.err
done
cat gpurun_out/k2_contention.jsonl
timeout 1200 python -m pytest tests/test_kernels_gpu.py tests/test_engine_gpu.py -x -q -m gpu > gpurun_out/pytest_k2dyn.log 2>&1; echo "pytest rc $?"
tail -3 gpurun_out/pytest_k2dyn.log
