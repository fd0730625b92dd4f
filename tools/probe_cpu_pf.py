"""Split-master CPU AdamW (the pool's kernel at c4max) alone and beside H2D + D2H DMA, for the software
prefetch distance in SH_CPU_PF (read once per process: run one process per value).  28 host-DRAM bytes
per element.  Prints one JSON line.  A measurement script, not product code."""
import json
import os
import sys
import threading
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_sunwqyhxw22_b200 import sh  # noqa: E402

N = 1 << 28
hi = torch.empty(N, dtype=torch.int16).pin_memory().numpy().view(np.uint16)
lo = torch.empty(N, dtype=torch.int16).pin_memory().numpy().view(np.uint16)
m = torch.zeros(N, dtype=torch.float32).pin_memory().numpy()
v = torch.zeros(N, dtype=torch.float32).pin_memory().numpy()
g = torch.empty(N, dtype=torch.float32).pin_memory().numpy()
g[:] = np.random.default_rng(1).standard_normal(N, dtype=np.float32) * 1e-3
hi[:] = 0x3c00
lo[:] = 0
sc = sh.adam_scalars(1.5e-4, 0.9, 0.999, 1e-8, 0.01, 1)
DB = 1 << 30
dev = torch.device("cuda:0")
hsrc, hdst = torch.empty(DB, dtype=torch.uint8).pin_memory(), torch.empty(DB, dtype=torch.uint8).pin_memory()
dsrc, ddst = torch.empty(DB, dtype=torch.uint8, device=dev), torch.empty(DB, dtype=torch.uint8, device=dev)
s1, s2 = torch.cuda.Stream(dev), torch.cuda.Stream(dev)


def adam(T, n=N):
    sh.op_adamw_split_cpu(hi, lo, m, v, g, n, n // 2, sc, threads=T)


def alone(T):
    adam(T)
    best = 1e9
    for _ in range(4):
        t = time.perf_counter()
        adam(T)
        best = min(best, time.perf_counter() - t)
    return 28.0 * N / best / 1e9


def with_dma(T, seconds=4.0):
    stop = threading.Event()
    res = {}

    def dma():
        a0, b0 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a1, b1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a0.record(s1)
        a1.record(s2)
        k = 0
        while not stop.is_set():
            with torch.cuda.stream(s1):
                dsrc.copy_(hsrc, non_blocking=True)
            with torch.cuda.stream(s2):
                hdst.copy_(ddst, non_blocking=True)
            k += 1
            if k % 2 == 0:
                s1.synchronize()
                s2.synchronize()
        b0.record(s1)
        b1.record(s2)
        torch.cuda.synchronize()
        res["h2d"] = k * DB / (a0.elapsed_time(b0) / 1e3) / 1e9
        res["d2h"] = k * DB / (a1.elapsed_time(b1) / 1e3) / 1e9

    th = threading.Thread(target=dma)
    th.start()
    time.sleep(0.3)
    t, n = time.perf_counter(), 0
    while time.perf_counter() - t < seconds:
        adam(T)
        n += N
    dt = time.perf_counter() - t
    stop.set()
    th.join()
    a = 28.0 * n / dt / 1e9
    return {"adam": round(a, 1), "h2d": round(res["h2d"], 1), "d2h": round(res["d2h"], 1),
            "total": round(a + res["h2d"] + res["d2h"], 1)}


out = {"pf": int(os.environ.get("SH_CPU_PF", "0"))}
for T in (12, 16):
    out[f"alone_T{T}"] = round(alone(T), 1)
for T in (14, 16):
    out[f"dma_T{T}"] = with_dma(T)
print(json.dumps(out), flush=True)
