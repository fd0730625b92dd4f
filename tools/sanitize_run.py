"""Tiny windowed training for compute-sanitizer (memcheck / racecheck / synccheck / initcheck):
2 steps at window 1 (prefetch, K1 restage, K3, D2H, CPU Adam, K2 all run) in bf16 and fp32."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_sunwqyhxw22_b200 import sh  # noqa: E402
from tests._common import TINY, engine_run  # noqa: E402

import tempfile  # noqa: E402

for prec, attn in ((sh.SH_BF16_MIXED, "cublas"), (sh.SH_FP32, "cublas")):
    tr, losses, norms = engine_run(TINY, 2, 1, prec, attention=attn)
    print("precision", prec, "losses", losses, "norms", norms)
    tr.close()
# NEXT-3 executors (K4) through the one-rank NCCL DP path, and the NEXT-2 spill tier
tr, losses, _ = engine_run(dict(TINY, b=4), 2, 1, sh.SH_FP32, attention="cublas", executors=2,
                           flags=sh.SH_FLAG_TEST_DP_PATH, nccl_id=sh.nccl_unique_id())
print("executors+dp losses", losses)
tr.close()
with tempfile.TemporaryDirectory() as d:
    tr, losses, _ = engine_run(TINY, 2, 1, sh.SH_BF16_MIXED, attention="cublas", spill_dir=d, host_pin_budget_bytes=1)
    print("spill losses", losses)
    tr.close()
print("SANITIZE_RUN_OK")
