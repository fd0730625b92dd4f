"""Does the page size backing a pinned host buffer change the copy engines' rate on this box?

Allocates a 4 GiB anonymous mapping with MADV_HUGEPAGE (the engine's host store / landing buffers,
engine.cpp host_alloc) and one with MADV_NOHUGEPAGE, touches it, registers it with cudaHostRegister,
reports how much of it the kernel backed with 2 MiB pages (/proc/self/smaps AnonHugePages of that
range), then times 1 GiB H2D / D2H copies (cudaMemcpyAsync, CUDA events, best of 5).  Prints one
JSON line per mode.
"""
import ctypes
import json
import mmap
import os

import torch
from cuda.bindings import runtime as rt  # cuda-python

GiB = 1 << 30


def anon_huge_kb(addr, size):
    tot, inside = 0, False
    for ln in open("/proc/self/smaps"):
        parts = ln.split()
        if "-" in parts[0] and len(parts) > 1 and ":" not in parts[0]:
            lo, hi = (int(x, 16) for x in parts[0].split("-"))
            inside = lo < addr + size and hi > addr
        elif inside and ln.startswith("AnonHugePages:"):
            tot += int(parts[1])
    return tot


def ck(r):
    err = r[0] if isinstance(r, tuple) else r
    assert err == rt.cudaError_t.cudaSuccess, r
    return r[1] if isinstance(r, tuple) and len(r) > 1 else None


def main():
    torch.cuda.init()
    dev = torch.empty(GiB, dtype=torch.uint8, device="cuda")
    st = torch.cuda.Stream()
    for mode in ("hugepage", "nohugepage"):
        mm = mmap.mmap(-1, 4 * GiB, flags=mmap.MAP_PRIVATE | mmap.MAP_ANONYMOUS)
        mm.madvise(mmap.MADV_HUGEPAGE if mode == "hugepage" else mmap.MADV_NOHUGEPAGE)
        buf = (ctypes.c_char * (4 * GiB)).from_buffer(mm)
        addr = ctypes.addressof(buf)
        ctypes.memset(addr, 1, 4 * GiB)
        huge = anon_huge_kb(addr, 4 * GiB) * 1024 / (4 * GiB)
        ck(rt.cudaHostRegister(addr, 4 * GiB, 0))
        res = {"mode": mode, "huge_frac": round(huge, 3)}
        for name, kind in (("h2d", rt.cudaMemcpyKind.cudaMemcpyHostToDevice),
                           ("d2h", rt.cudaMemcpyKind.cudaMemcpyDeviceToHost)):
            best = 0.0
            for rep in range(6):
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                off = (rep % 3) * GiB
                a.record(st)
                if name == "h2d":
                    ck(rt.cudaMemcpyAsync(dev.data_ptr(), addr + off, GiB, kind, st.cuda_stream))
                else:
                    ck(rt.cudaMemcpyAsync(addr + off, dev.data_ptr(), GiB, kind, st.cuda_stream))
                b.record(st)
                torch.cuda.synchronize()
                if rep:
                    best = max(best, GiB / (a.elapsed_time(b) / 1e3) / 1e9)
            res[name + "_gbs"] = round(best, 2)
        ck(rt.cudaHostUnregister(addr))
        del buf
        mm.close()
        print(json.dumps(res), flush=True)
    thp = {k: open(f"/sys/kernel/mm/transparent_hugepage/{k}").read().strip() for k in ("enabled", "defrag")}
    print(json.dumps({"thp": thp, "pid": os.getpid()}))


if __name__ == "__main__":
    main()
