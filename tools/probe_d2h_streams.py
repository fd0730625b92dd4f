"""Does splitting a D2H copy over two streams (two copy engines) raise its rate while the CPU AdamW
saturates host DRAM?  The pool's split AdamW runs on 16 threads (tools/probe_cpu_pf.py's arrays) while
H2D copies run on one stream and D2H on 1 / 2 / 4 streams; prints one JSON line per D2H stream count.
A measurement script, not product code."""
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
g[:] = 1e-3
hi[:] = 0x3c00
sc = sh.adam_scalars(1.5e-4, 0.9, 0.999, 1e-8, 0.01, 1)
DB = 1 << 30
dev = torch.device("cuda:0")
hsrc, hdst = torch.empty(DB, dtype=torch.uint8).pin_memory(), torch.empty(DB, dtype=torch.uint8).pin_memory()
dsrc, ddst = torch.empty(DB, dtype=torch.uint8, device=dev), torch.empty(DB, dtype=torch.uint8, device=dev)
s_h2d = torch.cuda.Stream(dev)
s_d2h = [torch.cuda.Stream(dev) for _ in range(4)]


def run(k, seconds=4.0, cpu=True):
    stop = threading.Event()
    res = {}

    def adam():
        n = 0
        t = time.perf_counter()
        while not stop.is_set():
            sh.op_adamw_split_cpu(hi, lo, m, v, g, N, N // 2, sc, threads=16)
            n += N
        res["adam"] = 28.0 * n / (time.perf_counter() - t) / 1e9

    th = threading.Thread(target=adam)
    if cpu:
        th.start()
        time.sleep(0.3)
    torch.cuda.synchronize()
    a = torch.cuda.Event(enable_timing=True)
    b = torch.cuda.Event(enable_timing=True)
    a.record(s_d2h[0])
    for s in s_d2h[1:k]:
        s.wait_event(a)
    t_end = time.perf_counter() + seconds
    reps = 0
    part = DB // k
    while time.perf_counter() < t_end:
        with torch.cuda.stream(s_h2d):
            dsrc.copy_(hsrc, non_blocking=True)
        for j in range(k):
            with torch.cuda.stream(s_d2h[j]):
                hdst[j * part:(j + 1) * part].copy_(ddst[j * part:(j + 1) * part], non_blocking=True)
        reps += 1
        if reps % 2 == 0:
            torch.cuda.synchronize()
    for s in s_d2h[1:k]:
        s_d2h[0].wait_stream(s)
    b.record(s_d2h[0])
    torch.cuda.synchronize()
    stop.set()
    if cpu:
        th.join()
    return {"d2h_streams": k, "cpu_adam": cpu, "d2h_gbs": round(reps * DB / (a.elapsed_time(b) / 1e3) / 1e9, 1),
            "adam_gbs": round(res.get("adam", 0.0), 1)}


for cpu in (False, True):
    for k in (1, 2, 4):
        print(json.dumps(run(k, cpu=cpu)), flush=True)
