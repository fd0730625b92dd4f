"""GPU-box probe. A measurement script, not product code.

Records host facts (cores, NUMA, RAM, memlock, THP), PCIe H2D/D2H/bidirectional bandwidth from
pinned memory, cudaHostRegister cost, host DRAM triad bandwidth, and the stream-memop attribute
used by the engine's readiness flags.  Output: gpurun_out/probe.json (+ raw text).
"""
import json, os, subprocess, time, ctypes, sys
out = {}
def sh(cmd):
    try:
        return subprocess.run(cmd, shell=True, capture_output=True, text=True, timeout=120).stdout
    except Exception as e:
        return str(e)
out["nvidia_smi_L"] = sh("nvidia-smi -L")
out["topo"] = sh("nvidia-smi topo -m")
out["gpu_q"] = sh("nvidia-smi --query-gpu=pcie.link.gen.max,pcie.link.gen.current,pcie.link.width.max,memory.total --format=csv")
out["nproc"] = sh("nproc").strip()
out["lscpu"] = sh("lscpu")
out["numa"] = sh("cat /sys/devices/system/node/node*/meminfo | grep MemTotal")
out["meminfo"] = sh("head -5 /proc/meminfo")
out["memlock"] = sh("ulimit -l").strip()
out["thp"] = sh("cat /sys/kernel/mm/transparent_hugepage/enabled")
out["lsblk"] = sh("lsblk -d -o NAME,SIZE,ROTA,MODEL")
out["cgroup_mem"] = sh("cat /sys/fs/cgroup/memory.max 2>/dev/null; cat /sys/fs/cgroup/cpu.max 2>/dev/null")
import torch
dev = torch.device("cuda:0")
torch.cuda.init()
props = torch.cuda.get_device_properties(0)
out["gpu"] = str(props)
def bw(n_bytes, direction, reps=5):
    h = torch.empty(n_bytes, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(n_bytes, dtype=torch.uint8, device=dev)
    best = 1e9
    for _ in range(reps):
        s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
        s.record()
        if direction == "h2d": d.copy_(h, non_blocking=True)
        else: h.copy_(d, non_blocking=True)
        e.record(); torch.cuda.synchronize()
        best = min(best, s.elapsed_time(e) / 1e3)
    return n_bytes / best / 1e9
for sz in (64 << 20, 256 << 20, 1 << 30):
    out[f"h2d_GBs_{sz>>20}MiB"] = bw(sz, "h2d")
    out[f"d2h_GBs_{sz>>20}MiB"] = bw(sz, "d2h")
# bidirectional on one GPU
n = 1 << 30
h1 = torch.empty(n, dtype=torch.uint8, pin_memory=True); h2 = torch.empty(n, dtype=torch.uint8, pin_memory=True)
d1 = torch.empty(n, dtype=torch.uint8, device=dev); d2 = torch.empty(n, dtype=torch.uint8, device=dev)
s1 = torch.cuda.Stream(); s2 = torch.cuda.Stream()
best = 1e9
for _ in range(5):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    with torch.cuda.stream(s1): d1.copy_(h1, non_blocking=True)
    with torch.cuda.stream(s2): h2.copy_(d2, non_blocking=True)
    torch.cuda.synchronize(); best = min(best, time.perf_counter() - t0)
out["bidir_total_GBs"] = 2 * n / best / 1e9
# cudaHostRegister cost for 8 GiB of malloc'ed memory
cudart = ctypes.CDLL("libcudart.so.12") if os.path.exists("/usr/local/cuda/lib64/libcudart.so.12") else None
try:
    libc = ctypes.CDLL("libc.so.6")
    libc.aligned_alloc.restype = ctypes.c_void_p
    nb = 8 << 30
    p = libc.aligned_alloc(ctypes.c_size_t(1 << 21), ctypes.c_size_t(nb))
    libc.memset(ctypes.c_void_p(p), 0, ctypes.c_size_t(nb))
    t0 = time.perf_counter()
    rc = torch.cuda.cudart().cudaHostRegister(p, nb, 0)
    out["host_register_8GiB_s"] = time.perf_counter() - t0
    out["host_register_rc"] = str(rc)
except Exception as e:
    out["host_register_err"] = repr(e)
# host DRAM triad (C + OpenMP compiled here)
src = r'''
#include <stdio.h>
#include <stdlib.h>
#include <omp.h>
int main(){ size_t n = (size_t)1<<28; double *a=aligned_alloc(64,n*8),*b=aligned_alloc(64,n*8),*c=aligned_alloc(64,n*8);
#pragma omp parallel for
for(size_t i=0;i<n;i++){a[i]=1;b[i]=2;c[i]=0;}
double best=1e9; for(int r=0;r<5;r++){ double t=omp_get_wtime();
#pragma omp parallel for
for(size_t i=0;i<n;i++) c[i]=a[i]+1.5*b[i];
t=omp_get_wtime()-t; if(t<best)best=t;}
printf("%d %.2f\n", omp_get_max_threads(), 3.0*n*8/best/1e9); return 0; }
'''
open("/tmp/triad.c", "w").write(src)
out["triad_build"] = sh("gcc -O3 -march=native -fopenmp /tmp/triad.c -o /tmp/triad 2>&1")
out["triad_all"] = sh("/tmp/triad")
out["triad_half"] = sh(f"OMP_NUM_THREADS={max(1, os.cpu_count()//2)} /tmp/triad")
out["triad_8"] = sh("OMP_NUM_THREADS=8 /tmp/triad")
# stream mem ops attribute (CU_DEVICE_ATTRIBUTE_CAN_USE_STREAM_MEM_OPS_V1 = 92? query via cuda-python)
try:
    from cuda import cuda as cu
    cu.cuInit(0)
    err, d = cu.cuDeviceGet(0)
    for name in ("CU_DEVICE_ATTRIBUTE_CAN_USE_STREAM_MEM_OPS_V1", "CU_DEVICE_ATTRIBUTE_CAN_USE_STREAM_WAIT_VALUE_NOR_V1",
                 "CU_DEVICE_ATTRIBUTE_CAN_USE_64_BIT_STREAM_MEM_OPS_V1", "CU_DEVICE_ATTRIBUTE_CAN_USE_HOST_POINTER_FOR_REGISTERED_MEM",
                 "CU_DEVICE_ATTRIBUTE_HOST_NATIVE_ATOMIC_SUPPORTED", "CU_DEVICE_ATTRIBUTE_PAGEABLE_MEMORY_ACCESS",
                 "CU_DEVICE_ATTRIBUTE_HOST_REGISTER_SUPPORTED"):
        a = getattr(cu.CUdevice_attribute, name, None)
        if a is not None:
            out[name] = cu.cuDeviceGetAttribute(a, d)[1]
except Exception as e:
    out["cuda_python_err"] = repr(e)
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/probe.json", "w"), indent=1)
for k, v in out.items():
    if k not in ("lscpu", "topo"):
        print(k, "=", v if not isinstance(v, str) else v.strip()[:300])
