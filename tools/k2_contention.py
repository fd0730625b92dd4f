"""K2 (fused AdamW) at one h=4096 layer (201 M elements, 30 B/elem) alone and beside what runs next to
it in the live step: a D2H of host-layer gradients on the copy engine, H2D + D2H together, a K3 on
another stream.  CUDA events on K2's stream, L2 flushed before each rep, median of reps.
Schedule / build selected by the environment of the process (SH_K2_SCHED=static|dyn, SH_K2_IMPL=ldg3 ...),
so run one process per variant:
    for v in "SH_K2_SCHED=static" "SH_K2_SCHED=dyn" "SH_K2_SCHED=dyn SH_K2_IMPL=ldg3"; do
        env $v python tools/k2_contention.py "$v"; done
"""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_sunwqyhxw22_b200 import sh  # noqa: E402


def main():
    tag = sys.argv[1] if len(sys.argv) > 1 else os.environ.get("SH_K2_SCHED", "default")
    pk = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                     "MEASURED_PEAKS.json")))["hbm_gbs"]
    n = 201_379_840
    d = torch.device("cuda")
    sc = sh.adam_scalars(1.5e-4, 0.9, 0.999, 1e-8, 0.01, 3)
    p = torch.randn(n, device=d) * 0.02
    m = torch.zeros(n, device=d)
    v = torch.zeros(n, device=d)
    g = torch.randn(n, device=d) * 1e-3
    o16 = torch.empty(n, dtype=torch.int16, device=d)
    g2 = torch.randn(n, device=d)
    acc = torch.zeros(1, dtype=torch.float64, device=d)
    host = torch.empty(512 << 20, dtype=torch.uint8, pin_memory=True)
    host2 = torch.empty(512 << 20, dtype=torch.uint8, pin_memory=True)
    dsrc = torch.empty(512 << 20, dtype=torch.uint8, device=d)
    ddst = torch.empty(512 << 20, dtype=torch.uint8, device=d)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=d)
    ks = torch.cuda.Stream()
    d2h, h2d, k3s = torch.cuda.Stream(), torch.cuda.Stream(), torch.cuda.Stream()

    def side(mode):
        if "d2h" in mode:
            with torch.cuda.stream(d2h):
                for _ in range(2):
                    host.copy_(dsrc, non_blocking=True)
        if "h2d" in mode:
            with torch.cuda.stream(h2d):
                for _ in range(2):
                    ddst.copy_(host2, non_blocking=True)
        if "k3" in mode:
            with torch.cuda.stream(k3s):
                sh.op_sumsq_gpu(g2, n, acc, stream=k3s)

    for rnd, mode in enumerate(("alone", "d2h", "h2d+d2h", "k3", "k3+d2h") * 2):
        ts = []
        for rep in range(13):
            flush.zero_()
            torch.cuda.synchronize()
            side(mode)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            with torch.cuda.stream(ks):
                a.record(ks)
                sh.op_adamw_gpu(p, m, v, g, o16, None, n, n // 2, sc, stream=ks)
                b.record(ks)
            torch.cuda.synchronize()
            if rep >= 3:
                ts.append(a.elapsed_time(b))
        ts.sort()
        ms = ts[len(ts) // 2]
        print(json.dumps({"variant": tag, "pass": rnd // 5, "mode": mode, "ms": round(ms, 4), "gbs": round(30 * n / ms / 1e6, 1),
                          "frac": round(30 * n / ms / 1e6 / pk, 4), "min_ms": round(ts[0], 4)}), flush=True)


if __name__ == "__main__":
    main()
