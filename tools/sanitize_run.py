"""Tiny windowed training for compute-sanitizer (memcheck / racecheck / synccheck / initcheck):
2 steps at window 1 (prefetch, K1 restage, K3, D2H, CPU Adam, K2 all run) in bf16 and fp32."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_sunwqyhxw22_b200 import sh  # noqa: E402
from tests._common import TINY, engine_run  # noqa: E402

for prec, attn in ((sh.SH_BF16_MIXED, "cublas"), (sh.SH_FP32, "cublas")):
    tr, losses, norms = engine_run(TINY, 2, 1, prec, attention=attn)
    print("precision", prec, "losses", losses, "norms", norms)
    tr.close()
print("SANITIZE_RUN_OK")
