#!/bin/bash
# The GPU-box runs behind the round-2 evidence in profiles/ (run under gpurun, one GPU):
#   bash tools/gpu_runs.sh verify     build + smoke() + the default bench + the c4max full-size parity test
#   bash tools/gpu_runs.sh full       build + smoke() + K2 schedule microbench + default bench + whole `pytest -m gpu`
#   bash tools/gpu_runs.sh k2         K2 schedule / build variants beside the step's concurrent traffic
#   bash tools/gpu_runs.sh ncu        ncu iso captures of K1-K4 + the c4max launch list (tools/ncu_c4max.sh)
#   bash tools/gpu_runs.sh cpu_pf     CPU AdamW prefetch probe + DMA page-size probe + c4max A/B
#   bash tools/gpu_runs.sh next4      NEXT-4 fixed-byte window vs the layer-count ring on C2
#   bash tools/gpu_runs.sh hybrid     R28 hybrid-update GPU tests + c4max A/B over the number of hybrid layers
#   bash tools/gpu_runs.sh ab NAME|ENV|ARGS ...   c4max A/B (tools/ab_c4max.sh, L = 112)
# Outputs land in gpurun_out/; the summaries worth keeping are copied to profiles/ by hand.
set -u
mkdir -p gpurun_out

build() { python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }; }
smoke() { python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc $?"; }
bench_default() {
  timeout 1500 python bench.py --trace-out gpurun_out/trace_default.json > gpurun_out/bench_default.json \
    2> gpurun_out/bench_default.err; echo "bench rc $?"
  python - <<'PY'
import json
d = json.loads(open("gpurun_out/bench_default.json").read().strip().splitlines()[-1])
print(d["value"], d["e2e"]["value"], d["runs"]["samples_per_s"], d["resident_fit"]["frac_model_tflops"], d["roofline"]["frac"],
      d["host_dram"]["achieved_gbs"], d["host_dram"]["frac"], d["compute_stream"]["stall_frac"], d["config"]["window"],
      d["config"]["ring_slots"])
PY
}
k2() {
  rm -f gpurun_out/k2_contention.jsonl
  for v in "SH_K2_SCHED=dyn" "SH_K2_SCHED=static" "SH_K2_IMPL=dyn2" "SH_K2_SCHED=static SH_K2_IMPL=ldg3"; do
    env $v timeout 300 python tools/k2_contention.py "$v" >> gpurun_out/k2_contention.jsonl 2>> gpurun_out/k2_contention.err
  done
  grep '"pass": 1' gpurun_out/k2_contention.jsonl
}
next4() {
  for spec in "ring|" "bytes5|--ring-bytes-slots 5" "bytes6|--ring-bytes-slots 6" "bytes8|--ring-bytes-slots 8"; do
    IFS='|' read -r NAME ARGS <<< "$spec"
    timeout 900 python bench.py --config c2 --window 4 --steps 10 --no-resident --no-cpu-baseline $ARGS \
      > gpurun_out/next4_$NAME.json 2> gpurun_out/next4_$NAME.err
    python - "$NAME" <<'PY'
import json, sys
n = sys.argv[1]
try:
    d = json.loads(open(f"gpurun_out/next4_{n}.json").read().strip().splitlines()[-1])
    c = d["config"]
    print(n, round(d["value"], 2), "e2e", round(d["e2e"]["value"], 2), "slots", c["ring_slots"], "ring_GB",
          round((c.get("ring_bytes") or 0) / 1e9, 3), "stall", round(d["compute_stream"]["stall_frac"], 3), flush=True)
except Exception as e:
    print(n, "FAILED", e, open(f"gpurun_out/next4_{n}.err").read()[-800:], flush=True)
PY
  done
}

case "${1:-}" in
  verify)
    smoke; bench_default
    timeout 1500 python -m pytest tests/test_fullsize_c4max_gpu.py -x -q -m gpu > gpurun_out/pytest_c4max.log 2>&1
    echo "c4max rc $?"; tail -1 gpurun_out/pytest_c4max.log ;;
  full)
    smoke; k2; bench_default
    timeout 2400 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu_full.log 2>&1
    echo "pytest rc $?"; tail -1 gpurun_out/pytest_gpu_full.log ;;
  k2) build; k2 ;;
  ncu) bash tools/ncu_c4max.sh ;;
  cpu_pf)
    build
    timeout 600 python tools/probe_dma_pages.py > gpurun_out/dma_pages.jsonl 2>&1; cat gpurun_out/dma_pages.jsonl
    rm -f gpurun_out/cpu_pf.jsonl
    for pf in 0 256 512 1024; do
      SH_CPU_PF=$pf timeout 600 python tools/probe_cpu_pf.py >> gpurun_out/cpu_pf.jsonl 2>> gpurun_out/cpu_pf.err
    done
    cat gpurun_out/cpu_pf.jsonl
    bash tools/ab_c4max.sh 112 "pf0|SH_CPU_PF=0|" "pf512|SH_CPU_PF=512|" ;;
  next4) build; next4 ;;
  hybrid)
    smoke
    timeout 1200 python -m pytest tests/test_hybrid_gpu.py tests/test_kernels_gpu.py tests/test_engine_gpu.py -x -q -m gpu \
      > gpurun_out/pytest_hybrid.log 2>&1; echo "pytest rc $?"; tail -15 gpurun_out/pytest_hybrid.log
    grep -q "passed" gpurun_out/pytest_hybrid.log && ! grep -q "failed\|error" gpurun_out/pytest_hybrid.log || exit 1
    bash tools/ab_c4max.sh 112 "hyb0||" "hyb4||--hybrid-layers 4" "hyb8||--hybrid-layers 8" "hyb12||--hybrid-layers 12" ;;
  ab) shift; build; bash tools/ab_c4max.sh 112 "$@" ;;
  hybrid2)
    build
    bash tools/ab_c4max.sh 112 "hyb0b||" "hyb6s2|SH_HYB_STAGING=2|--hybrid-layers 6"
    timeout 2400 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu_full.log 2>&1
    echo "pytest rc $?"; tail -1 gpurun_out/pytest_gpu_full.log ;;
  *) sed -n 2,10p "$0"; exit 2 ;;
esac
