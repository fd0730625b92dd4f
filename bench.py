"""Benchmark of the STRONGHOLD working-window engine on B200 (one JSON line on rank 0).

  python bench.py [--gpus N --steps K --warmup W] [--config c2|c3|tiny] [--batch B] [--window w]
  python bench.py --impl reference ...     # the CPU oracle, timed on this box's host cores

Metric (BASELINE.json): samples/s at max trainable size per B200; host-link GB/s vs peak.
Workload (N=1, default `--config c4max`): BASELINE.json configs[3] at the size the metric is quoted
at, "max trainable size per B200": a depth-scaled GPT (h 4096, 32 heads, seq 1024, V 50304) of
L = 112 layers (22.8 B params; pinned -- what this pool's 196 GB hosts and the HBM hold together, warming
up with 42 GPU-optimised layers beside a 26-slot ring; a smaller host falls back to its own maximum),
fp32 p/m/v 273 GB > 180 GB of HBM, the host-optimised layers' split fp32 master + Adam m, v in pinned host RAM (12 B/param), bf16 mixed
precision, batch 16 per GPU, window auto-tuned by the paper's model (P1/P2) plus the eq. 3
CPU-throughput constraint.  `--config c4` is the same width at L = L_max(host RAM) with a 2-layer
warm-up set (round-1 default), `c2` configs[1] (GPT-2 XL-shaped 1.5B), `c3` configs[2] (10B), `tiny`
configs[0].  A "step" is one full
training iteration through every §8(a) row: prefetch H2D, K1 restage, per-layer K3, grad D2H,
CPU AdamW, K2 (and, outside the hot path, the GPT block compute that drives it).

Timing: W untimed warm-up steps; K timed steps bracketed by barrier + synchronize; CUDA events
on the engine's compute stream; the end event is recorded after sh_synchronize (all copies and
all CPU Adam updates of the K steps complete); max over ranks.  Per-step traffic (GBs of weights,
grads and states) is far larger than the 126 MB L2, so no explicit flush is needed.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

CONFIGS = {
    # name: (L, h, nh, s, V, default batch, default window, description)
    "tiny": (4, 256, 4, 128, 512, 2, 2, "BASELINE configs[0]: tiny GPT 4x256, seq 128"),
    "c2": (48, 1600, 25, 1024, 50304, 16, 4, "BASELINE configs[1]: GPT-2 XL-shaped 1.5B (48 x 1600, seq 1024)"),
    "c3": (48, 4096, 32, 1024, 50304, 16, -1, "BASELINE configs[2]: GPT-style ~10B (48 x 4096, seq 1024)"),
    # depth-scaled h=4096 GPT with L = L_max(host RAM); on a 196 GB host that is
    # 77 layers = 15.7 B params, fp32 params + Adam states 188 GB > 180 GB of HBM, host store 12 B/param
    # (fp32-fetch mode, no bf16 shadow)
    "c4": (0, 4096, 32, 1024, 50304, 16, -1, "BASELINE configs[3]: depth-scaled GPT h4096, L = L_max(host RAM), "
                                            "fp32 states > 180 GB HBM, auto-tuned window"),
    # the largest model HBM + host RAM hold together: GPU-optimised layers keep no host copy, so the run
    # warms up with the first C4MAX_W0 layers already in HBM beside a decoupled C4MAX_RING0-slot ring
    # (the configuration R27 settles on) and only layers >= C4MAX_W0 need host blocks
    "c4max": (0, 4096, 32, 1024, 50304, 16, -1, "max trainable size: depth-scaled GPT h4096, 112 layers "
                                                "(22.8 B params), auto-tuned window"),
}
C4MAX_W0 = 42
C4MAX_HYB_W0_COST = 2  # the hybrid update's 3 HBM staging buffers (10 B/param each) displace ~2 GPU layers
C4MAX_RING0 = 26
# the depth the default line is quoted at: 112 x 4096 = 22.8 B params, fp32 p/m/v 273 GB (> 180 GB of HBM);
# 70 host layers (170 GB of pinned state) beside the 42-layer warm-up GPU set on this pool's 196 GB hosts
# (118 layers do not fit the HBM next to the activations; profiles/r02_ab_c4max_L112.txt).  A box with
# less RAM falls back to its own L_max and says so (config.layers_pinned).
C4MAX_LAYERS = 112
# bf16 host layout: the split master (R25: hi plane = the bf16 compute copy, fetched at 2 B/param;
# 12 B/param of host RAM) for every config; --fetch-fp32 1 / --bf16-shadow select the round-1 layouts
FETCH_FP32_DEFAULT: set = set()
CPU_HARD_DEFAULT = {"c3", "c4", "c4max"}   # autotune with the eq. 3 CPU-throughput constraint (R19)
# autotune with the B200 extensions of the window model by default (R22/R23): landing-ring
# growth, GPU set filling the HBM a decoupled ring leaves, late bf16 host shadows (C4: 7.30 -> 7.92
# samples/s, profiles/r01_bench_default_c4_v3.json vs r01_bench_c4_tuned_coupled.json)
TUNED_DEFAULT = {"c3", "c4"}
# c4max: no host RAM is left to grow the landing ring, so the decoupled ring is sized as a gradient pool
# for the backward backlog and the GPU set fills the rest of the HBM (R27; profiles/r02_ab4:
# 44-47 GPU layers / ring 20-26 beat the coupled 38 / 39 by 3.5 %)
FILL_DEFAULT = {"c4max"}
SETTLE_MAX = 10   # at most this many untimed settle steps after the autotuner's window change
RUNS = 3          # the K timed steps are timed as RUNS consecutive segments (median / geomean reported)


def mem_available() -> int:
    for ln in open("/proc/meminfo"):
        if ln.startswith("MemAvailable:"):
            return int(ln.split()[1]) * 1024
    return 0


def host_pages() -> dict:
    """Huge-page backing of the process's host memory while the engine holds its pinned store (the host
    store is mmap'ed with MADV_HUGEPAGE: whether the kernel could back it with 2 MiB pages is a property
    of the box -- THP mode, fragmentation -- that the DMA rates may depend on)."""
    out = {}
    try:
        for ln in open("/proc/self/smaps_rollup"):
            k = ln.split(":")[0]
            if k in ("Rss", "AnonHugePages"):
                out[k.lower() + "_gb"] = int(ln.split()[1]) * 1024 / 1e9
    except OSError:
        pass
    for k in ("enabled", "defrag"):
        try:
            out["thp_" + k] = open(f"/sys/kernel/mm/transparent_hugepage/{k}").read().strip()
        except OSError:
            pass
    return out


def layer_n_pad(h: int) -> int:
    """Elements of one GPT block's packed layout (every tensor padded to 128 elements)."""
    return sum((n + 127) // 128 * 128 for n in (h, h, 3 * h * h, 3 * h, h * h, h, h, h, 4 * h * h, 4 * h, 4 * h * h, h))


def ring_bytes_of(mc, bf16: bool, slots: float) -> int:
    """Device bytes of `slots` largest-layer slots of the fixed-byte ring (engine.cpp slot_sz:
    the compute copy and the fp32 gradient half, each 256-B aligned)."""
    n = layer_n_pad(mc.hidden)
    cb = 2 if bf16 else 4
    slot = (cb * n + 255) // 256 * 256 + (4 * n + 255) // 256 * 256
    return int(slots * slot)


def shm_free() -> int:
    try:
        st = os.statvfs("/dev/shm")
        return st.f_bavail * st.f_frsize
    except OSError:
        return 0


def c4_layers(h: int, ring: int, w0: int = 2, margin_gb: float = 8.0, ranks_sharing: int = 1,
              budget: int | None = None) -> int:
    """Deepest h-wide GPT whose host store (12 B/param, per-layer 2 MiB-aligned blocks for layers
    >= w0, plus `ring` landing buffers per rank) fits in MemAvailable - margin (or `budget`)."""
    avail = budget if budget is not None else mem_available()
    n_pad = sum((n + 127) // 128 * 128 for n in (h, h, 3 * h * h, 3 * h, h * h, h, h, h, 4 * h * h, 4 * h, 4 * h * h, h))
    per_layer = (12 * n_pad + (1 << 21) - 1) // (1 << 21) * (1 << 21)
    budget = avail - int(margin_gb * (1 << 30)) - ranks_sharing * ring * 4 * n_pad
    return max(w0 + 1, budget // per_layer + w0)
METRIC = "samples/s at max trainable size per B200; host-link GB/s vs peak"
PROBE_H2D_GBS = 55.58   # profiles/r01_probe_box.json, pinned 1 GiB H2D, best of 5
PROBE_D2H_GBS = 57.01
PROBE_HOST_TRIAD_GBS = 143.43  # profiles/r01_probe_box.json, 16-thread STREAM triad (no RFO counted)
# The engine's real host-DRAM mix -- the pool's split-master CPU AdamW (16 B read + 12 B written per
# element) running concurrently with H2D + D2H DMA on pinned memory: the highest total host-DRAM
# throughput measured over thread counts and software-prefetch distances (profiles/r02_cpu_pf.jsonl,
# tools/probe_cpu_pf.py: 14 threads, prefetch 1024: Adam 142.5 + H2D 27.7 + D2H 27.7 GB/s).  Round-2
# first probe without the prefetch (profiles/r02_host_mix.json): 184.7; the 16-thread STREAM triad: 143.
PROBE_HOST_MIX_GBS = 197.9


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    FIELDS = "clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown," \
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown," \
             "clocks_event_reasons.sw_power_cap"

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 7:
                continue
            try:
                sm.append(float(f[0]))
                mx.append(float(f[1]))
            except ValueError:
                continue
            for n, v in zip(names, f[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        return {"sm_mhz": float(np.median(sm)), "sm_max_mhz": max(mx), "reasons": sorted(reasons),
                "samples": len(sm)}


def k2_traffic(elems_per_launch: float):
    """DRAM read+write bytes of one K2 launch: the per-element figure of the committed ncu --set full
    capture (tools/ncu_kernels.sh -> tools/ncu_iso_summary.py) times this bench's elements per launch."""
    for name in ("r02_ncu_iso_kernels.json", "r01_ncu_iso_kernels.json"):
        try:
            per = json.load(open(os.path.join(ROOT, "profiles", name)))["k2_adamw"]["dram_bytes_per_elem"]
        except Exception:  # noqa: BLE001
            continue
        return per * elems_per_launch, "profiles/" + name
    return None, None


def oracle_sample(L, h, nh, s, V, b, seed=1234):
    """Bounded CPU-oracle sample of the workload: one block's fwd+bwd at batch 1 and its AdamW, the
    head's fwd+bwd at batch 1 and the resident AdamW, each timed once.  One training step of the full
    model at batch b costs L (b t_fb + t_adam) + b t_head + t_adam_res (the AdamW runs once per STEP,
    not per sample); returns (seconds per step, parts)."""
    from oracle import gpt_oracle as O
    import synth
    P = [a.astype(np.float64) for a in synth.init_layer(seed, 0, L, h)]
    R = [a.astype(np.float64) for a in synth.init_resident(seed, V, s, h)]
    tok = synth.tokens(0, 1, s, V)
    opt = O.AdamWConfig()
    x = R[0][tok[:, :-1]] + R[1][None, :s]
    t0 = time.perf_counter()
    y, cache = O.block_fwd(x, P, nh)
    dx, grads = O.block_bwd(np.ones_like(y) * 1e-3, cache, P)
    t_fb = time.perf_counter() - t0
    t0 = time.perf_counter()
    for k, (p, g) in enumerate(zip(P, grads)):
        O.adamw_update(p, g, np.zeros_like(p), np.zeros_like(p), 1, opt, p.ndim == 2)
    t_adam = time.perf_counter() - t0
    t0 = time.perf_counter()
    O.forward_backward(O.GPTConfig(0, h, nh, s, V), [], R, tok)
    t_head = time.perf_counter() - t0
    t0 = time.perf_counter()
    for p in R:
        O.adamw_update(p, p, np.zeros_like(p), np.zeros_like(p), 1, opt, True)
    t_adam_res = time.perf_counter() - t0
    per_step = L * (b * t_fb + t_adam) + b * t_head + t_adam_res
    return per_step, dict(t_fb=t_fb, t_adam=t_adam, t_head=t_head, t_adam_res=t_adam_res)


def oracle_desc(L, b, parts):
    return (f"one block fwd+bwd at batch 1 ({parts['t_fb']:.2f} s) and its AdamW ({parts['t_adam']:.2f} s), the head "
            f"fwd+bwd at batch 1 ({parts['t_head']:.2f} s) and the resident AdamW ({parts['t_adam_res']:.2f} s), numpy "
            f"fp64, extrapolated to one step: L x (b x fwd+bwd + AdamW) + b x head + resident AdamW, L={L}, b={b}")


def spill_line(args, r, K):
    """NEXT-2: the spill tier's disk traffic per step and its rate vs the same O_DIRECT io_uring path probed on
    a fresh file in the same directory (sh_spill_probe)."""
    from paper_conf_sc_sunwqyhxw22_b200 import sh
    st0, st1 = r["st0"], r["st1"]
    rd, wr = st1["spill_read_bytes"] - st0["spill_read_bytes"], st1["spill_write_bytes"] - st0["spill_write_bytes"]
    io_ms = st1["spill_io_ms"] - st0["spill_io_ms"]
    try:
        probe = sh.spill_probe(args.spill_dir, 2 << 30)
    except Exception as e:  # noqa: BLE001
        probe = {"error": str(e)}
    out = {"dir": args.spill_dir, "layers": st1["spilled_layers"], "bytes": st1["spill_bytes"],
           "o_direct": bool(st1["spill_direct"]), "io_uring": bool(st1["spill_uring"]),
           "read_bytes_per_step": rd / K, "write_bytes_per_step": wr / K,
           "disk_gbs_while_busy": (rd + wr) / (io_ms / 1e3) / 1e9 if io_ms > 0 else None,
           "disk_gbs_per_step": (rd + wr) / (r["ms"] / 1e3) / 1e9, "probe": probe}
    if "read_gbs" in probe and out["disk_gbs_while_busy"]:
        out["frac_of_probe"] = (rd + wr) / (io_ms / 1e3) / 1e9 / (
            (rd * probe["read_gbs"] + wr * probe["write_gbs"]) / max(1, rd + wr))
    return out


def blas_threads():
    try:
        from threadpoolctl import threadpool_info
        return max(int(i.get("num_threads", 1)) for i in threadpool_info()) or os.cpu_count()
    except Exception:
        return os.cpu_count()


def run_reference(args, cfgname):
    L, h, nh, s, V, b, w, desc = CONFIGS[cfgname]
    b = args.batch or b
    if args.layers:
        L = args.layers
    if L == 0:  # same depth rule as the CUDA arm (L_max of this host's RAM; c4max pinned)
        L = c4_layers(h, args.grad_ring or 8, w0=C4MAX_W0 if cfgname == "c4max" else 2,
                      ranks_sharing=int(os.environ.get("LOCAL_WORLD_SIZE", "1")))
        if cfgname == "c4max":
            L = min(L, C4MAX_LAYERS)
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    times = []
    for i in range(args.warmup + args.steps):
        per_step, parts = oracle_sample(L, h, nh, s, V, b)
        if i >= args.warmup:
            times.append(per_step)
    per = float(np.mean(times))
    val = b / per
    line = {"impl": "reference", "metric": METRIC, "value": val,
            "unit": "samples/s", "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": per * 1e3, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "f64", "data": "synthetic",
            "config": {"workload": cfgname, "description": desc, "layers": L, "hidden": h, "heads": nh,
                       "batch_per_gpu": b, "seq": s, "vocab": V},
            "cpu_baseline": {"value": val, "unit": "samples/s", "cores": blas_threads(), "kind": "oracle",
                             "sample": "per timed step: " + oracle_desc(L, b, parts)},
            "e2e": {"value": val, "unit": "samples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="sh", choices=["sh", "reference"])
    ap.add_argument("--config", default="c4max", choices=sorted(CONFIGS))
    ap.add_argument("--batch", type=int, default=0)
    ap.add_argument("--window", type=int, default=-2, help="-2: config default, -1: autotune, L: resident")
    ap.add_argument("--precision", default="bf16", choices=["bf16", "fp32"])
    ap.add_argument("--cpu-threads", type=int, default=0)
    ap.add_argument("--grad-ring", type=int, default=0)
    ap.add_argument("--no-resident", action="store_true", help="skip the all-resident comparison run")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--fetch-fp32", type=int, default=-1, help="1: fp32 master in host RAM, fp32 over the link + K1")
    ap.add_argument("--bf16-shadow", action="store_true", help="fp32 master + bf16 shadow in host RAM (14 B/param)")
    ap.add_argument("--init-threads", type=int, default=16)
    ap.add_argument("--layers", type=int, default=0, help="override the depth (c4: L_max(host RAM))")
    ap.add_argument("--trace-out", default="", help="write a Chrome trace of the last profiled step")
    ap.add_argument("--resident-fit-layers", type=int, default=-1,
                    help="c3/c4: also time the all-resident model of the same width with this depth "
                         "(SURVEY §8(d): the >=85%% bar denominator; -1: 36 for h=4096, 0: skip)")
    ap.add_argument("--fp-only", action="store_true",
                    help="NEXT-4: time FP-only streaming passes (KD-teacher inference, PAPER.md:357-368)")
    ap.add_argument("--slice-fetch", action="store_true",
                    help="N>1: NEXT-1 slice H2D + NVLink all-gather (SH_FLAG_SLICE_FETCH)")
    ap.add_argument("--attention", default="auto", choices=["auto", "flash", "cublas"],
                    help="attention core of the GPT driver (outside the hot path)")
    ap.add_argument("--cpu-hard", type=int, default=-1, help="1: autotune with the eq. 3 CPU constraint")
    ap.add_argument("--spill-dir", default="", help="NEXT-2: directory of the file-backed tier (PAPER.md:219-221)")
    ap.add_argument("--host-pin-gb", type=float, default=0.0,
                    help="NEXT-2: pinned host-store budget in GB (layers beyond it spill to --spill-dir)")
    ap.add_argument("--ablate-alloc", action="store_true",
                    help="Fig. 14 ablation: cudaMalloc/cudaFree per prefetch instead of the reserved ring")
    ap.add_argument("--grow-landing", action="store_true",
                    help="autotune may decouple the ring by growing the landing ring (SH_FLAG_GROW_LANDING)")
    ap.add_argument("--no-decouple", action="store_true", help="autotune keeps the ring coupled to the GPU set")
    ap.add_argument("--fill-gpu", action="store_true", help="decoupled autotune fills HBM with GPU-optimised layers")
    ap.add_argument("--late-shadow", action="store_true", help="fp32-fetch mode: bf16 host shadows after the autotune")
    ap.add_argument("--plain-autotune", action="store_true",
                    help="c3/c4: autotune without --grow-landing/--fill-gpu/--late-shadow (the round-1 default)")
    ap.add_argument("--ring", type=int, default=0, help="ring size (prefetch distance + 1): with a fixed --window, or the "
                                                        "warm-up ring of an autotuned run")
    ap.add_argument("--warmup-window", type=int, default=0,
                    help="GPU-optimised layers during an autotuned run's warm-up (c4max default: %d)" % C4MAX_W0)
    ap.add_argument("--sync-cpu", action="store_true",
                    help="Fig. 14 ablation: one CPU Adam at a time, inline when a layer's grads land (no pool)")
    ap.add_argument("--spill-evict", action="store_true", help="NEXT-2: drop spilled layers from the page cache")
    ap.add_argument("--dp-test-host-collective", action="store_true",
                    help="TEST ONLY (N > 1 ranks on ONE GPU): gloo bootstrap, every rank on cuda:0, the engine's "
                         "collectives through SH_FLAG_TEST_HOST_COLLECTIVE -- exercises the multi-rank bench "
                         "orchestration where NCCL cannot run (not a performance number)")
    ap.add_argument("--hybrid-layers", type=int, default=0,
                    help="R28: the lowest K host-optimised layers are updated on the GPU (states stay in host RAM)")
    ap.add_argument("--ring-bytes-slots", type=float, default=0.0,
                    help="NEXT-4 fixed-byte window: ring_bytes = this many largest-layer slots (param + grad halves)")
    ap.add_argument("--executors", type=int, default=1,
                    help="NEXT-3: K multi-stream executors (micro-batches of batch/K on K streams, PAPER.md:227-242)")
    args = ap.parse_args()
    if args.config in TUNED_DEFAULT and not args.plain_autotune and args.window in (-2, -1):
        args.grow_landing = args.fill_gpu = args.late_shadow = True
    if args.config in FILL_DEFAULT and not args.plain_autotune and args.window in (-2, -1):
        args.fill_gpu = True
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args, args.config)

    import torch
    import torch.distributed as dist
    from paper_conf_sc_sunwqyhxw22_b200 import gpt as G
    from paper_conf_sc_sunwqyhxw22_b200 import sh
    from paper_conf_sc_sunwqyhxw22_b200.trainer import ModelConfig, StrongholdTrainer
    import synth

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    host_coll = args.dp_test_host_collective and world > 1
    if host_coll:
        local = 0  # every rank on the one GPU
    torch.cuda.set_device(local)
    tdev = torch.device("cpu") if host_coll else torch.device("cuda", local)  # torch.distributed tensors

    def fresh_nccl_id():
        # an ncclUniqueId bootstraps ONE communicator: every engine context (the timed run, the
        # resident-fit run) gets its own, created on rank 0 and broadcast over torch.distributed
        idt = torch.zeros(128, dtype=torch.uint8, device=tdev)
        if rank == 0:
            raw = os.urandom(128) if host_coll else sh.nccl_unique_id()
            idt.copy_(torch.frombuffer(bytearray(raw), dtype=torch.uint8))
        dist.broadcast(idt, 0)
        return bytes(idt.cpu().numpy().tobytes())

    nccl_id = None
    if world > 1:
        if host_coll:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        nccl_id = fresh_nccl_id()

    L, h, nh, s, V, b0, w0, desc = CONFIGS[args.config]
    b = args.batch or b0
    w = w0 if args.window == -2 else args.window
    # data parallel: one shared /dev/shm host store per box when /dev/shm can hold it, else a
    # private replica per rank with the host RAM divided between the ranks of the box
    local_world = int(os.environ.get("LOCAL_WORLD_SIZE", world))
    use_shm = world > 1
    if world > 1:
        flag = torch.tensor([1 if host_coll or shm_free() > 0.8 * mem_available() else 0], dtype=torch.int64,
                            device=tdev)
        dist.broadcast(flag, 0)
        use_shm = bool(flag.item())
    if args.layers and L != 0:
        L = args.layers  # depth override (e.g. the resident-fit comparison model)
    if L == 0:
        w0h = (C4MAX_W0 - (C4MAX_HYB_W0_COST if args.hybrid_layers else 0)) if args.config == "c4max" else 2
        if args.layers:
            L = args.layers
        elif args.config == "c4max":
            L = min(C4MAX_LAYERS, c4_layers(h, args.grad_ring or 8, w0=args.warmup_window or w0h,
                                            ranks_sharing=local_world))
        elif not use_shm and world > 1:
            L = c4_layers(h, args.grad_ring or 8, budget=mem_available() // local_world)
        else:
            L = c4_layers(h, args.grad_ring or 8, ranks_sharing=local_world)
        if world > 1:  # every rank must build the same model
            lt = torch.tensor([L], dtype=torch.int64, device=tdev)
            dist.broadcast(lt, 0)
            L = int(lt.item())
    prec = sh.SH_BF16_MIXED if args.precision == "bf16" else sh.SH_FP32
    mc = ModelConfig(L, h, nh, s, V)
    K, W = args.steps, args.warmup

    fetch32 = args.fetch_fp32 == 1 or (args.fetch_fp32 == -1 and args.config in FETCH_FP32_DEFAULT)
    cpu_hard = args.cpu_hard == 1 or (args.cpu_hard == -1 and args.config in CPU_HARD_DEFAULT)
    # c3/c4 are host-RAM bound: 8 landing buffers (measured on C4: 4 -> 6.80, 8 -> 7.08, 12 -> 7.51
    # samples/s at L = 83, 82, 80; profiles/r01_bench_c4_ring*.json)
    grad_ring = args.grad_ring or (8 if args.config in ("c3", "c4", "c4max") else 0)

    shm_name = None
    cpu_threads = args.cpu_threads
    import hashlib
    if world > 1:
        if use_shm:
            shm_name = "sh_" + hashlib.sha1(nccl_id).hexdigest()[:16]  # one host store for the box
        cpu_threads = cpu_threads or max(1, (os.cpu_count() or 1) // local_world)

    first_run = [True]

    def run(window, e2e: bool, mc=mc):
        L = mc.n_layers
        nid, shm = nccl_id, shm_name
        if world > 1 and not first_run[0]:
            nid = fresh_nccl_id()
            if shm_name:
                shm = "sh_" + hashlib.sha1(nid).hexdigest()[:16]
        first_run[0] = False
        t_init = time.perf_counter()
        flags = sh.SH_FLAG_PROFILE | (sh.SH_FLAG_FETCH_FP32 if fetch32 else 0) | \
            (sh.SH_FLAG_CPU_HARD | (0 if args.no_decouple else sh.SH_FLAG_DECOUPLE) if cpu_hard else 0) | \
            (sh.SH_FLAG_SLICE_FETCH if args.slice_fetch else 0) | \
            (sh.SH_FLAG_SPILL_EVICT if args.spill_evict else 0) | \
            (sh.SH_FLAG_ABLATE_ALLOC if args.ablate_alloc else 0) | (sh.SH_FLAG_SYNC_CPU if args.sync_cpu else 0) | \
            (sh.SH_FLAG_GROW_LANDING if args.grow_landing else 0) | (sh.SH_FLAG_FILL_GPU if args.fill_gpu else 0) | \
            (sh.SH_FLAG_LATE_SHADOW if args.late_shadow else 0) | (sh.SH_FLAG_BF16_SHADOW if args.bf16_shadow else 0) | \
            (sh.SH_FLAG_TEST_HOST_COLLECTIVE if host_coll else 0)
        tr = StrongholdTrainer(mc, batch=b, window=window, precision=prec, device=local,
                               flags=flags, world_size=world, rank=rank, nccl_id=None if host_coll else nid,
                               cpu_threads=cpu_threads, grad_ring_depth=grad_ring, shm_name=shm,
                               warmup_steps=W if window == -1 else 5, init_threads=args.init_threads,
                               attention=args.attention, executors=args.executors,
                               ring_slots=args.ring or (C4MAX_RING0 if args.config == "c4max" and window == -1 else 0),
                               spill_dir=args.spill_dir or None, host_pin_budget_bytes=int(args.host_pin_gb * 1e9),
                               warmup_window=(args.warmup_window or
                                              (C4MAX_W0 - (C4MAX_HYB_W0_COST if args.hybrid_layers else 0)
                                               if args.config == "c4max" else 0))
                               if window == -1 else 0,
                               hybrid_layers=args.hybrid_layers,
                               ring_bytes=ring_bytes_of(mc, prec == sh.SH_BF16_MIXED, args.ring_bytes_slots) if args.ring_bytes_slots > 0 else 0)
        attn_used = "flash_attn 2.8 (library, deterministic bwd)" if tr.flash is not None else "cuBLAS batched + softmax"
        t_init = time.perf_counter() - t_init
        # tokens: step t uses synth.tokens(t) (rank-offset seeds for DP)
        # an autotuned run changes its window (and with the extensions its landing ring and host
        # shadows) at the end of warm-up step W; S more untimed steps let the new configuration reach
        # its steady state (GPU-set uploads, ring refill) so the timed steps measure it, not the switch
        S_max = SETTLE_MAX if window == -1 else 0
        host = torch.stack([torch.from_numpy(synth.tokens(t + 1000 * rank, b, s, V)) for t in range(W + S_max + K)])
        host = host.pin_memory()
        dev = host.to(f"cuda:{local}")
        step_fn = tr.forward_only if args.fp_only else tr.step_device

        def one(t):
            with torch.cuda.stream(tr.stream):  # ordered after the previous step's reads of tok_dev
                tr.tok_dev.copy_(dev[t], non_blocking=True)
            step_fn()

        def mark():
            e = torch.cuda.Event(enable_timing=True)
            e.record(tr.stream)
            return e

        for t in range(W):
            one(t)
        # settle (autotuned runs switch window / landing ring / shadows at the end of warm-up): untimed
        # steps until two consecutive step times agree within 3 % -- step i's time is read once step
        # i+1 is issued, so the host never starves the GPU to measure it
        t = W
        settle_ms = []
        if S_max:
            marks = [mark()]
            while t < W + S_max:
                one(t)
                t += 1
                marks.append(mark())
                if len(marks) >= 3:
                    marks[-2].synchronize()
                    settle_ms.append(marks[-3].elapsed_time(marks[-2]))
                    if len(settle_ms) >= 2 and abs(settle_ms[-1] - settle_ms[-2]) <= 0.03 * settle_ms[-2]:
                        break
        S = t - W
        tr.engine.synchronize()
        st0 = tr.engine.stats()
        l0 = sh.kernel_launches() + G.kernel_launches()
        # K timed steps in R segments (the runs of the protocol: median / geomean over >= 3)
        R = max(1, min(RUNS, K // 3))
        bounds = [t + (K * r) // R for r in range(R + 1)]
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        with ClockSampler(local) as clk:
            seg = [mark()]
            for r in range(R):
                for tt in range(bounds[r], bounds[r + 1]):
                    one(tt)
                if r < R - 1:
                    seg.append(mark())
            tr.engine.synchronize()  # every copy and CPU update of the K steps
            seg.append(mark())
            torch.cuda.synchronize()
        ms = seg[0].elapsed_time(seg[-1])
        seg_ms = [seg[r].elapsed_time(seg[r + 1]) for r in range(R)]
        seg_sps = [b * world * (bounds[r + 1] - bounds[r]) / (seg_ms[r] / 1e3) for r in range(R)]
        launches = sh.kernel_launches() + G.kernel_launches() - l0
        st1 = tr.engine.stats()
        loss = tr.loss()
        e2e_ms = None
        if e2e and not args.fp_only:
            if world > 1:
                dist.barrier()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(tr.stream)
            for tt in range(W + S, W + S + K):
                tr.step(host[tt])  # public API: pinned host tokens -> H2D, step, loss -> host
            tr.engine.synchronize()
            e1.record(tr.stream)
            torch.cuda.synchronize()
            e2e_ms = e0.elapsed_time(e1)
        prof = tr.engine.profile() if window != L else None
        trace = tr.engine.trace()
        st2 = tr.engine.stats()
        hostmem = host_pages()
        if args.trace_out and rank == 0:
            # Chrome trace (chrome://tracing / Perfetto) of the last profiled step: Fig. 4 analogue
            tid = {"fp": 1, "bp": 1, "k2_adamw": 1, "h2d_fp": 2, "h2d_bp": 2, "d2h_grad": 3, "k1_stage": 4,
                   "k3_sumsq": 5, "cpu_adam": 6, "h2d_wait_cpu": 7}
            ev = [{"name": f"{e['kind']} L{e['layer']}", "ph": "X", "pid": 0, "tid": tid[e["kind"]],
                   "ts": e["start_ms"] * 1e3, "dur": (e["end_ms"] - e["start_ms"]) * 1e3} for e in trace]
            names = {1: "compute stream", 2: "H2D copy engine", 3: "D2H copy engine", 4: "K1 stage stream",
                     5: "K3 (D2H stream)", 6: "CPU Adam pool (host clock)", 7: "H2D issuer waiting on CPU Adam"}
            ev += [{"name": "thread_name", "ph": "M", "pid": 0, "tid": k, "args": {"name": v}} for k, v in names.items()]
            with open(args.trace_out + (f".w{window}" if window != w else ""), "w") as f:
                json.dump({"traceEvents": ev, "displayTimeUnit": "ms"}, f)
        tr.close()
        return dict(ms=ms, e2e_ms=e2e_ms, st0=st0, st1=st1, loss=loss, launches=launches, clocks=clk.summary(),
                    hostmem=hostmem,
                    init_s=t_init, prof=prof, st2=st2, attn=attn_used, seg_sps=seg_sps, settle_ms=settle_ms, S=S)

    r = run(w, not args.no_e2e)
    res = None
    if not args.no_resident and w != L and args.config not in ("c3", "c4", "c4max"):
        res = run(L, False)
    fit = None
    fit_layers = args.resident_fit_layers if args.resident_fit_layers >= 0 else (36 if h == 4096 else 0)
    if args.config in ("c3", "c4", "c4max") and fit_layers > 0 and not args.no_resident:
        mc_fit = ModelConfig(fit_layers, h, nh, s, V)
        fit = run(fit_layers, False, mc_fit)
        fit["tflops"] = b * world * K / (fit["ms"] / 1e3) * s * mc_fit.flops_per_token() / 1e12

    def gmax(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=tdev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    ms = gmax(r["ms"])
    e2e_ms = gmax(r["e2e_ms"]) if r["e2e_ms"] is not None else None
    res_ms = gmax(res["ms"]) if res else None
    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return
    st0, st1 = r["st0"], r["st1"]
    d = {k: st1[k] - st0[k] for k in ("h2d_bytes", "d2h_bytes", "h2d_busy_ms", "d2h_busy_ms",
                                      "h2d_profiled_bytes", "d2h_profiled_bytes", "cpu_adam_ms",
                                      "cpu_adam_elems", "cpu_adam_shadow_elems", "cpu_wait_ms", "k2_ms_sum",
                                      "k2_bytes_sum", "k2_samples", "k3_ms_sum", "k3_bytes_sum", "k3_samples")}
    # host-DRAM bytes of the CPU AdamW: 28 B/element (r p, m, v, g + w p, m, v), +2 for the elements
    # whose layer also has a bf16 shadow (counted by the engine per element)
    adam_bytes = 28 * d["cpu_adam_elems"] + 2 * d["cpu_adam_shadow_elems"]
    host_dram_bytes = adam_bytes + d["h2d_bytes"] + d["d2h_bytes"]
    step_ms = ms / K
    samples = b * world * K / (ms / 1e3)
    peak, peak_kind = measured_peaks()
    k2_gbs = d["k2_bytes_sum"] / (d["k2_ms_sum"] / 1e3) / 1e9 if d["k2_ms_sum"] > 0 else None
    k2_tr, k2_tr_src = k2_traffic(d["k2_bytes_sum"] / max(1, d["k2_samples"]) / (30 if prec else 32))
    k3_gbs = d["k3_bytes_sum"] / (d["k3_ms_sum"] / 1e3) / 1e9 if d["k3_ms_sum"] > 0 else None
    h2d_gbs = d["h2d_profiled_bytes"] / (d["h2d_busy_ms"] / 1e3) / 1e9 if d["h2d_busy_ms"] > 0 else None
    d2h_gbs = d["d2h_profiled_bytes"] / (d["d2h_busy_ms"] / 1e3) / 1e9 if d["d2h_busy_ms"] > 0 else None
    flops_tok = mc.flops_per_token()
    tokens_s = samples * s
    if args.fp_only:  # FP-only passes: 2 flop/param/token for the layers + the head forward
        flops_tok = 2 * mc.n_layers * mc.params_per_layer() + 2 * h * V
    line = {
        "metric": METRIC if not args.fp_only else "samples/s, FP-only streaming inference (NEXT-4)",
        "value": samples, "unit": "samples/s", "n_gpus": world, "steps": K, "warmup": W,
        "ms_per_step": step_ms, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
        "dtype": "bf16" if prec == sh.SH_BF16_MIXED else "f32", "data": "synthetic",
        "config": {"workload": args.config, "description": desc, "layers": L,
                   "layers_pinned": (L == C4MAX_LAYERS) if args.config == "c4max" and not args.layers else None,
                   "hidden": h, "heads": nh, "seq": s,
                   "vocab": V, "params": mc.n_params(), "batch_per_gpu": b, "global_batch": b * world,
                   "window": r["st1"]["window"], "ring_slots": r["st1"]["n_slots"],
                   "ring_bytes": r["st1"].get("ring_bytes"),
                   "fixed_byte_ring": args.ring_bytes_slots or None,
                   "hybrid_layers": args.hybrid_layers or None,
                   "window_mode": ("autotuned (P1/P2" + (" + eq.3 CPU throughput, ring decoupled from the GPU set"
                                                         if cpu_hard else "") + ")") if w == -1 else "fixed",
                   "precision": "bf16_mixed" if prec else "fp32",
                   "gpt_driver_attention": r["attn"],
                   "parallelism": f"dp{world}" + (" (TEST: host collective, all ranks on one GPU)" if host_coll else ""),
                   "executors": args.executors,
                   "ablation": [k for k, v in (("alloc", args.ablate_alloc), ("sync_cpu", args.sync_cpu),
                                               ("cpu_threads", args.cpu_threads)) if v] or None,
                   "spill": spill_line(args, r, K) if args.spill_dir else None,
                   "host_store": ("one shared /dev/shm store, rank-sliced offload + CPU Adam" if shm_name else
                                  "private per rank") if world > 1 else "private",
                   "numa": {"nodes": r["st1"]["numa_nodes"],
                            "policy": ("auto", "split", "local", "interleave", "none")[r["st1"]["numa_policy"]],
                            "gpu_node": r["st1"]["numa_gpu_node"], "pinned_workers": r["st1"]["numa_pinned_workers"],
                            "bound_bytes": r["st1"]["numa_bound_bytes"]},
                   "states": (("split fp32 master (bf16 hi plane = compute copy + 16-bit lo plane), m, v in pinned "
                               "host RAM, 12 B/param") if prec == sh.SH_BF16_MIXED and not fetch32 and not args.bf16_shadow
                              else "fp32 master/m/v in pinned host RAM" + ("" if not st1["shadow_layers"] else " + bf16 shadow")),
                   "fetch": ("hi plane of the split master (bf16, 2 B/param)" if prec == sh.SH_BF16_MIXED and not fetch32
                             and not args.bf16_shadow else "bf16 shadow" if args.bf16_shadow else
                             f"bf16 shadow for {st1['shadow_layers']} of {L - st1['window']} host layers (late "
                             "shadows), fp32 master + K1 cast on the GPU for the rest" if st1["shadow_layers"] else
                             "fp32 master, K1 cast on GPU" if prec == sh.SH_BF16_MIXED else "fp32 master"),
                   "grad_landing_buffers": r["st1"]["landing_buffers"], "host_store_bytes": r["st1"]["host_bytes"],
                   "states_bytes_fp32_p_m_v": 12 * mc.n_params(),
                   "l2": "no flush: per-step traffic (GBs) >> 126 MB L2",
                   "settle_steps": r["S"], "settle_step_ms": r["settle_ms"]},
        "runs": {"n": len(r["seg_sps"]), "samples_per_s": r["seg_sps"], "median": float(np.median(r["seg_sps"])),
                 "geomean": float(np.exp(np.mean(np.log(r["seg_sps"])))),
                 "note": "the K timed steps as consecutive segments of one process (the last one includes the "
                         "drain of the CPU updates); value = all K steps"},
        "tokens_per_s": tokens_s,
        "model_tflops": tokens_s * flops_tok / 1e12,
        "final_loss": r["loss"],
        "host_memory": r.get("hostmem"),
        "host_link": {
            "h2d_bytes_per_step": d["h2d_bytes"] / K, "d2h_bytes_per_step": d["d2h_bytes"] / K,
            "h2d_gbs_per_transfer": h2d_gbs, "d2h_gbs_per_transfer": d2h_gbs,
            "h2d_peak_gbs": PROBE_H2D_GBS, "d2h_peak_gbs": PROBE_D2H_GBS,
            "h2d_frac": h2d_gbs / PROBE_H2D_GBS if h2d_gbs else None,
            "h2d_step_gbs": d["h2d_bytes"] / (ms / 1e3) / 1e9, "d2h_step_gbs": d["d2h_bytes"] / (ms / 1e3) / 1e9,
            "d2h_frac": d2h_gbs / PROBE_D2H_GBS if d2h_gbs else None,
            "h2d_busy_frac_of_step": d["h2d_busy_ms"] / ms, "d2h_busy_frac_of_step": d["d2h_busy_ms"] / ms,
            "h2d_overlap_with_compute": r["st2"]["h2d_overlap_frac"],
            "d2h_overlap_with_compute": r["st2"]["d2h_overlap_frac"],
            "peak_source": "profiles/r01_probe_box.json (pinned 1 GiB copies)"},
        # compute-stream stall of the last profiled step: step time minus the union of
        # the layer compute intervals and K2 on the compute stream (engine CUDA events)
        "compute_stream": {"step_ms": r["st2"]["last_step_ms"], "busy_ms": r["st2"]["compute_busy_ms"],
                           "stall_ms": r["st2"]["last_step_ms"] - r["st2"]["compute_busy_ms"],
                           "stall_frac": (1 - r["st2"]["compute_busy_ms"] / r["st2"]["last_step_ms"])
                           if r["st2"]["last_step_ms"] > 0 else None},
        "cpu_adam": {"threads": st1["cpu_threads"], "elems_per_step": d["cpu_adam_elems"] / K,
                     "thread_ms_per_step": d["cpu_adam_ms"] / K,
                     "dram_gbs": adam_bytes / (d["cpu_adam_ms"] / 1e3 / st1["cpu_threads"]) / 1e9
                     if d["cpu_adam_ms"] > 0 else None,
                     "prefetch_wait_ms_per_step": d["cpu_wait_ms"] / K,
                     "host_dram_triad_peak_gbs": PROBE_HOST_TRIAD_GBS,
                     "note": "dram_gbs counts the AdamW's 28 B/param (+2 where a bf16 shadow is written) while its "
                             "threads run; the copy engines' DMA shares the same host DRAM"},
        # whole-step host-DRAM roofline: the CPU AdamW's bytes (28 B/param fp32-fetch, 30 with the bf16
        # shadow: r p,m,v,g + w p,m,v [+ w shadow]) plus every DMA byte the copy engines move through
        # host DRAM, over the step time, against the probe's 16-thread triad
        "host_dram": {"bytes_per_step": host_dram_bytes / K,
                      "bytes_per_host_param": host_dram_bytes / max(1, d["cpu_adam_elems"]),
                      "achieved_gbs": host_dram_bytes / (ms / 1e3) / 1e9,
                      "peak_gbs": PROBE_HOST_MIX_GBS,
                      "frac": host_dram_bytes / (ms / 1e3) / 1e9 / PROBE_HOST_MIX_GBS,
                      "triad_gbs": PROBE_HOST_TRIAD_GBS,
                      "peak_source": "profiles/r02_cpu_pf.jsonl: the split-master CPU AdamW + H2D + D2H DMA "
                                     "concurrently (the engine's own mix), best total over thread counts and "
                                     "prefetch distances"},
        "roofline": {"kernel": "K2 fused AdamW: the per-layer launches of the GPU-optimised layers in the "
                               "backward + the resident-set launch at sh_step (CUDA events on their stream)",
                     "bound": "hbm", "achieved": k2_gbs,
                     "peak": peak, "unit": "GB/s", "frac": k2_gbs / peak if k2_gbs else None,
                     "traffic": k2_tr,
                     "traffic_source": (f"{k2_tr_src}: ncu --set full DRAM bytes/element of an isolated K2 launch "
                                        "(one h=4096 layer) x the K2 elements of one step") if k2_tr_src else None,
                     "traffic_per": "step",
                     "peak_source": peak_kind, "algorithmic_bytes_per_elem": 30 if prec else 32,
                     "bytes_per_step": d["k2_bytes_sum"] / max(1, d["k2_samples"]),
                     "k3_sumsq_gbs": k3_gbs, "k3_frac": k3_gbs / peak if k3_gbs else None},
        "gpu_launches": r["launches"],
        "clocks": r["clocks"],
        "init_s": r["init_s"],
    }
    if r["e2e_ms"] is not None:
        line["e2e"] = {"value": b * world * K / (e2e_ms / 1e3), "unit": "samples/s",
                       "h2d_bytes_per_step": b * (s + 1) * 4, "d2h_bytes_per_step": 4}
    if fit:
        line["resident_fit"] = {"layers": fit_layers, "window": fit_layers, "model_tflops": fit["tflops"],
                                "samples_per_s": b * world * K / (fit["ms"] / 1e3),
                                "frac_model_tflops": line["model_tflops"] / fit["tflops"],
                                "note": "same width, all layers GPU-resident (SURVEY §8(d) C4 bar: >= 0.85)"}
    if res:
        line["resident"] = {"window": L, "samples_per_s": b * world * K / (res_ms / 1e3),
                            "ms_per_step": res_ms / K, "frac_windowed_over_resident": res_ms / ms}
    if r["prof"]:
        p = r["prof"]
        # the engine's solver re-run on the profile of the TIMED steps (steady state at the tuned window),
        # with the same options the engine used after the warm-up
        rep = sh.solve_window(p["t_fp"], p["t_bp"], p["t_c2g"], p["t_g2c"], p["t_stage"], p["t_opt_gpu"],
                              p["t_opt_cpu"], p["t_async"], p["slot_bytes"], p["gstate_bytes"], p["fixed_bytes"],
                              p["s_avail"], p["duplex"], p["cpu_hard"], p["cpu_util_max"], p["decouple"],
                              p["fp_serial"], p["fill_gpu"])
        line["autotune"] = {"note": "solver re-run on the timed steps' profile", "window": rep["window"],
                            "ring_slots": rep["ring_slots"], "s_avail_gb": p["s_avail"] / 1e9,
                            "decouple": p["decouple"], "reason": rep["reason"], "eq3_ok": rep["eq3_ok"],
                            "eq3_min_slack_ms": rep["eq3_min_slack_ms"],
                            "t_fp_ms": float(np.median(p["t_fp"])), "t_bp_ms": float(np.median(p["t_bp"])),
                            "t_c2g_ms": float(np.median(p["t_c2g"])), "t_g2c_ms": float(np.median(p["t_g2c"])),
                            "t_opt_cpu_ms": float(np.median(p["t_opt_cpu"]))}
    if world == 1 and not args.no_cpu_baseline:
        per_step, parts = oracle_sample(L, h, nh, s, V, b)
        line["cpu_baseline"] = {"value": b / per_step, "unit": "samples/s", "cores": blas_threads(),
                                "kind": "oracle", "sample": oracle_desc(L, b, parts)}
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
