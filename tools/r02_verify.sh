#!/bin/bash
# Round-2 check of HEAD on one B200: build, smoke(), the default bench line, the c4max full-size parity test.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc $?"
tail -2 gpurun_out/smoke.log
timeout 1200 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; echo "bench rc $?"
tail -c 600 gpurun_out/bench_default.json
timeout 1500 python -m pytest tests/test_fullsize_c4max_gpu.py -x -q -m gpu > gpurun_out/pytest_c4max.log 2>&1; echo "c4max rc $?"
tail -3 gpurun_out/pytest_c4max.log
