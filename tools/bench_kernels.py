"""Isolated roofline of the hot-path kernels through the C-ABI op entry points (sh_op_*).

K2 (fused AdamW, 30 B/elem with bf16 out), K1 (cast, 6 B/elem), K3 (sum of squares, 4 B/elem)
at several sizes; CUDA events on the launching stream, warm-up first, L2 flushed between launches
by touching a 256 MB buffer.  Prints one JSON line per (kernel, size).
"""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_sunwqyhxw22_b200 import sh  # noqa: E402


def peak():
    p = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")
    return json.load(open(p))["hbm_gbs"] if os.path.exists(p) else 6650.0


def timeit(fn, reps=10):
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for _ in range(3):
        fn()
    ts = []
    for _ in range(reps):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    ts.sort()
    return ts[len(ts) // 2]


def main():
    pk = peak()
    sc = sh.adam_scalars(1.5e-4, 0.9, 0.999, 1e-8, 0.01, 3)
    for n in (1 << 22, 30_740_800 // 8 * 8, 201_379_840, 1 << 30):
        d = torch.device("cuda")
        p = torch.randn(n, device=d) * 0.02
        m = torch.zeros(n, device=d)
        v = torch.zeros(n, device=d)
        g = torch.randn(n, device=d) * 1e-3
        o16 = torch.empty(n, dtype=torch.int16, device=d)
        ms = timeit(lambda: sh.op_adamw_gpu(p, m, v, g, o16, None, n, n // 2, sc))
        print(json.dumps({"kernel": "K2", "n": n, "ms": ms, "gbs": 30 * n / ms / 1e6, "frac": 30 * n / ms / 1e6 / pk}))
        ms = timeit(lambda: sh.op_cast_bf16_gpu(p, o16, n))
        print(json.dumps({"kernel": "K1", "n": n, "ms": ms, "gbs": 6 * n / ms / 1e6, "frac": 6 * n / ms / 1e6 / pk}))
        out = torch.zeros(1, dtype=torch.float64, device=d)
        ms = timeit(lambda: sh.op_sumsq_gpu(g, n, out))
        print(json.dumps({"kernel": "K3", "n": n, "ms": ms, "gbs": 4 * n / ms / 1e6, "frac": 4 * n / ms / 1e6 / pk}))
        del p, m, v, g, o16
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
