"""Host-DRAM probe with the engine's real traffic mix (VERDICT r01 "make the host-side roofline honest").

A measurement script, not product code.  Measures on the GPU box, each alone and then concurrently:
  * the CPU AdamW of the pool (sh_op_adamw_cpu, the engine's AVX-512 kernel): 16 B read (p, m, v, g) +
    14 B written (p, m, v, bf16 shadow) per element, at several thread counts;
  * the copy engines: H2D + D2H from / to pinned host memory at the same time (the offload engine's
    two directions);
  * plain host streams (read-only sum, write-only memset, copy) for the DRAM ceiling.
Output: gpurun_out/host_mix.json.  Each concurrent number is the rate of one side while the other side
runs continuously for the whole measured window.
"""
import ctypes
import json
import os
import sys
import threading
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_sunwqyhxw22_b200 import sh  # noqa: E402

N = int(os.environ.get("MIX_N", 1 << 27))  # elements per Adam array (512 MiB fp32)
CH = 1 << 22
dev = torch.device("cuda:0")
out = {"n_elems": N, "nproc": os.cpu_count()}

p = torch.empty(N, dtype=torch.float32).pin_memory().numpy()
m = torch.empty(N, dtype=torch.float32).pin_memory().numpy()
v = torch.empty(N, dtype=torch.float32).pin_memory().numpy()
g = torch.empty(N, dtype=torch.float32).pin_memory().numpy()
s16 = torch.empty(N, dtype=torch.int16).pin_memory().numpy().view(np.uint16)
rng = np.random.default_rng(1)
p[:] = rng.standard_normal(N, dtype=np.float32) * 0.02
g[:] = rng.standard_normal(N, dtype=np.float32) * 1e-3
m[:] = 0
v[:] = 0
sc = sh.adam_scalars(1.5e-4, 0.9, 0.999, 1e-8, 0.01, 1)

DB = 1 << 30
hsrc = torch.empty(DB, dtype=torch.uint8).pin_memory()
hdst = torch.empty(DB, dtype=torch.uint8).pin_memory()
dsrc = torch.empty(DB, dtype=torch.uint8, device=dev)
ddst = torch.empty(DB, dtype=torch.uint8, device=dev)
s_h2d = torch.cuda.Stream(dev)
s_d2h = torch.cuda.Stream(dev)


def adam_once(threads):
    sh.op_adamw_cpu(p, m, v, g, s16, N, N // 2, sc, threads=threads)


def adam_rate(threads, reps=3):
    adam_once(threads)
    best = 1e9
    for _ in range(reps):
        t = time.perf_counter()
        adam_once(threads)
        best = min(best, time.perf_counter() - t)
    return 30.0 * N / best / 1e9


def dma_rate(seconds=2.0, h2d=True, d2h=True):
    """Copy-engine GB/s per direction over `seconds` of back-to-back 1 GiB copies."""
    torch.cuda.synchronize()
    ev = []
    t_end = time.perf_counter() + seconds
    n = 0
    a0 = torch.cuda.Event(enable_timing=True)
    b0 = torch.cuda.Event(enable_timing=True)
    a1 = torch.cuda.Event(enable_timing=True)
    b1 = torch.cuda.Event(enable_timing=True)
    a0.record(s_h2d)
    a1.record(s_d2h)
    while time.perf_counter() < t_end:
        if h2d:
            with torch.cuda.stream(s_h2d):
                dsrc.copy_(hsrc, non_blocking=True)
        if d2h:
            with torch.cuda.stream(s_d2h):
                hdst.copy_(ddst, non_blocking=True)
        n += 1
        if n % 2 == 0:
            s_h2d.synchronize()
            s_d2h.synchronize()
    b0.record(s_h2d)
    b1.record(s_d2h)
    torch.cuda.synchronize()
    r = {}
    if h2d:
        r["h2d"] = n * DB / (a0.elapsed_time(b0) / 1e3) / 1e9
    if d2h:
        r["d2h"] = n * DB / (a1.elapsed_time(b1) / 1e3) / 1e9
    return r


def adam_during(threads, fn):
    """Adam rate while fn() runs in another thread (Adam loops over chunks until fn returns)."""
    done = threading.Event()
    res = {}

    def bg():
        res["other"] = fn()
        done.set()

    th = threading.Thread(target=bg)
    th.start()
    time.sleep(0.2)
    elems = 0
    t = time.perf_counter()
    while not done.is_set():
        for b in range(0, N, N // 4):
            sh.op_adamw_cpu(p[b:], m[b:], v[b:], g[b:], s16[b:], N // 4, N // 8, sc, threads=threads)
            elems += N // 4
            if done.is_set():
                break
    dt = time.perf_counter() - t
    th.join()
    res["adam_GBs"] = 30.0 * elems / dt / 1e9
    return res


# plain host-DRAM streams (numpy with all cores is single-threaded; use the C triad-like ops via
# torch's parallel CPU kernels)
torch.set_num_threads(os.cpu_count())
a = torch.empty(1 << 28, dtype=torch.float32)
b = torch.empty(1 << 28, dtype=torch.float32)
a.fill_(1.0)
b.fill_(2.0)


def tmin(f, reps=4):
    f()
    best = 1e9
    for _ in range(reps):
        t = time.perf_counter()
        f()
        best = min(best, time.perf_counter() - t)
    return best


nb = 4 * (1 << 28)
out["host_read_GBs"] = nb / tmin(lambda: a.sum()) / 1e9
out["host_write_GBs"] = nb / tmin(lambda: a.fill_(3.0)) / 1e9
out["host_copy_GBs"] = 2 * nb / tmin(lambda: b.copy_(a)) / 1e9
out["host_triad_torch_GBs"] = 3 * nb / tmin(lambda: torch.add(a, b, alpha=1.5, out=b)) / 1e9
del a, b

out["dma_alone"] = dma_rate()
out["dma_h2d_alone"] = dma_rate(h2d=True, d2h=False)
out["dma_d2h_alone"] = dma_rate(h2d=False, d2h=True)
for T in (4, 8, 12, 14, 16):
    out[f"adam_alone_T{T}_GBs"] = adam_rate(T)
for T in (8, 12, 14, 16):
    r = adam_during(T, lambda: dma_rate(3.0))
    out[f"concurrent_T{T}"] = {"adam_GBs": r["adam_GBs"], "h2d_GBs": r["other"]["h2d"], "d2h_GBs": r["other"]["d2h"],
                               "host_total_GBs": r["adam_GBs"] + r["other"]["h2d"] + r["other"]["d2h"]}
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/host_mix.json", "w"), indent=1)
print(json.dumps(out, indent=1))
