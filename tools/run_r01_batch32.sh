#!/bin/bash
# Full GPU suite at HEAD (NUMA, fixed-byte window, heterogeneous units, full-size C4 parity, GPT-driver change).
mkdir -p gpurun_out
export SH_WAIT_TIMEOUT_S=600
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/pytest32.log 2>&1
tail -5 gpurun_out/pytest32.log
