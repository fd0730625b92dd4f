"""Launch each hot-path kernel a few times at one size (for `ncu --set full` captures).

  python tools/kernel_once.py [n]     # default n = 201_379_840 (one h=4096 layer, C3/C4)
K2 (AdamW, bf16 out, half the elements decayed), K1 (cast), K3 (sumsq), K4 (executor reduce,
2 executors) -- 3 launches each, in that order.
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_sunwqyhxw22_b200 import sh  # noqa: E402


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 201_379_840
    d = torch.device("cuda")
    sc = sh.adam_scalars(1.5e-4, 0.9, 0.999, 1e-8, 0.01, 3)
    p = torch.randn(n, device=d) * 0.02
    m = torch.zeros(n, device=d)
    v = torch.zeros(n, device=d)
    g = torch.randn(n, device=d) * 1e-3
    g2 = torch.randn(n, device=d) * 1e-3
    o16 = torch.empty(n, dtype=torch.int16, device=d)
    out = torch.zeros(1, dtype=torch.float64, device=d)
    for _ in range(3):
        sh.op_adamw_gpu(p, m, v, g, o16, None, n, n // 2, sc)
    for _ in range(3):
        sh.op_cast_bf16_gpu(p, o16, n)
    for _ in range(3):
        sh.op_sumsq_gpu(g, n, out)
    for _ in range(3):
        sh.op_exec_reduce_gpu(g, [g2], n, 0.5)
    torch.cuda.synchronize()
    print("done", n)


if __name__ == "__main__":
    main()
