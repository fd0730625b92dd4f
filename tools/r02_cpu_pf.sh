#!/bin/bash
# CPU AdamW software-prefetch distance: probe alone / beside DMA, then a c4max A/B.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 600 python tools/probe_dma_pages.py > gpurun_out/dma_pages.jsonl 2>&1; cat gpurun_out/dma_pages.jsonl
rm -f gpurun_out/cpu_pf.jsonl
for pf in 0 256 512 1024 0 512; do
  SH_CPU_PF=$pf timeout 600 python tools/probe_cpu_pf.py >> gpurun_out/cpu_pf.jsonl 2>> gpurun_out/cpu_pf.err
done
cat gpurun_out/cpu_pf.jsonl
bash tools/ab_c4max.sh 112 "pf0|SH_CPU_PF=0|" "pf512|SH_CPU_PF=512|" "pf0b|SH_CPU_PF=0|" "pf512b|SH_CPU_PF=512|"
