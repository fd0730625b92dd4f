#!/bin/bash
# Full check on one B200: build, K2 schedule microbench, the whole GPU suite, smoke(), the default bench.
mkdir -p gpurun_out
df -h / /tmp /dev/shm > gpurun_out/df.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc $?"
rm -f gpurun_out/k2_contention.jsonl
for v in "SH_K2_SCHED=dyn" "SH_K2_SCHED=static" "SH_K2_IMPL=dyn2"; do
  env $v timeout 300 python tools/k2_contention.py "$v" >> gpurun_out/k2_contention.jsonl 2>> gpurun_out/k2_contention.err
done
grep '"pass": 1' gpurun_out/k2_contention.jsonl
timeout 1500 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; echo "bench rc $?"
tail -c 300 gpurun_out/bench_default.json
timeout 2400 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu_full.log 2>&1; echo "pytest rc $?"
tail -3 gpurun_out/pytest_gpu_full.log
