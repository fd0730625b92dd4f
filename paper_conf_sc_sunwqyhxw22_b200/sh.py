"""ctypes binding of libsh.so (include/sh.h): argument marshalling only.

Every operation of the offload path runs in the native library (C++ engine + sm_100a kernels);
this module only converts Python values to the C structs and back.  There is no fallback: if
libsh.so is missing the import-time loader raises, and on a box without a GPU the engine calls
fail with the CUDA error the library reports.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIBDIR = os.path.join(_HERE, "lib")

SH_OK, SH_ERR_INVALID, SH_ERR_CUDA, SH_ERR_OOM_DEVICE, SH_ERR_OOM_HOST, SH_ERR_NCCL, SH_ERR_STATE, \
    SH_ERR_UNSUPPORTED = 0, -1, -2, -3, -4, -5, -6, -7
SH_FP32, SH_BF16_MIXED = 0, 1
SH_PRE, SH_POST = 0, 1
SH_READ_PARAM, SH_READ_M, SH_READ_V, SH_READ_COMPUTE, SH_READ_GRAD = 0, 1, 2, 3, 4
SH_FLAG_PROFILE, SH_FLAG_POISON, SH_FLAG_DUPLEX, SH_FLAG_SYNC_CPU, SH_FLAG_CPU_HARD, SH_FLAG_FETCH_FP32, \
    SH_FLAG_TEST_NO_COLLECTIVE, SH_FLAG_SLICE_FETCH, SH_FLAG_DELAY_INJECT, SH_FLAG_DECOUPLE, SH_FLAG_SPILL_EVICT, \
    SH_FLAG_TEST_DP_PATH, SH_FLAG_KEEP_GRADS, SH_FLAG_ABLATE_ALLOC, SH_FLAG_GROW_LANDING, SH_FLAG_FILL_GPU, \
    SH_FLAG_LATE_SHADOW = 1, 2, 4, 8, 16, 32, 64, 128, 256, 512, 1024, 2048, 4096, 8192, 16384, 32768, 65536
SH_FLAG_TEST_HOST_COLLECTIVE = 1 << 17
SH_FLAG_BF16_SHADOW = 1 << 18

# Every symbol include/sh.h declares (tests check the .so exports them all).
EXPORTS = ("sh_init", "sh_register_host_store", "sh_synchronize", "sh_destroy", "sh_forward_layer",
           "sh_backward_layer", "sh_resident", "sh_set_lr", "sh_step", "sh_solve_window",
           "sh_autotune_window", "sh_set_window", "sh_get_profile", "sh_read_layer", "sh_stats",
           "sh_last_error", "sh_abi_version", "sh_nccl_get_unique_id", "sh_adam_scalars_for",
           "sh_op_adamw_gpu", "sh_op_adamw_cpu", "sh_op_cast_bf16_gpu", "sh_op_cast_bf16_cpu",
           "sh_op_sumsq_gpu", "sh_kernel_launches", "sh_get_trace", "sh_forward_only_end", "sh_set_window_ring",
           "sh_executor_grads", "sh_op_exec_reduce_gpu", "sh_numa_topology", "sh_numa_plan",
           "sh_numa_worker_node", "sh_numa_node_of_pci", "sh_numa_bind_check", "sh_spill_probe", "sh_op_master_split_cpu",
           "sh_op_master_join_cpu", "sh_op_adamw_split_cpu", "sh_op_adamw_split_gpu")

# NUMA placement policies (sh_config.numa_policy, include/sh.h)
SH_NUMA_AUTO, SH_NUMA_SPLIT, SH_NUMA_LOCAL, SH_NUMA_INTERLEAVE, SH_NUMA_NONE = range(5)


class ShError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"sh status {status}: {msg}")
        self.status = status


class LayerShape(C.Structure):
    _fields_ = [("n_tensors", C.c_int32), ("numel", C.POINTER(C.c_int64)), ("weight_decay", C.POINTER(C.c_uint8))]


class Config(C.Structure):
    _fields_ = [("n_layers", C.c_int32), ("layers", C.POINTER(LayerShape)), ("resident", LayerShape),
                ("window", C.c_int32), ("precision", C.c_int32), ("lr", C.c_double), ("beta1", C.c_double),
                ("beta2", C.c_double), ("eps", C.c_double), ("weight_decay", C.c_double),
                ("max_grad_norm", C.c_double), ("device", C.c_int32), ("compute_stream", C.c_void_p),
                ("cpu_threads", C.c_int32), ("grad_ring_depth", C.c_int32), ("warmup_steps", C.c_int32),
                ("device_budget_bytes", C.c_int64), ("cpu_util_max", C.c_double), ("ring_slots", C.c_int32),
                ("world_size", C.c_int32), ("rank", C.c_int32),
                ("nccl_unique_id", C.c_void_p), ("flags", C.c_uint64), ("shm_name", C.c_char_p),
                ("n_executors", C.c_int32), ("spill_dir", C.c_char_p), ("host_pin_budget_bytes", C.c_int64),
                ("warmup_window", C.c_int32), ("numa_policy", C.c_int32), ("ring_bytes", C.c_int64),
                ("hybrid_layers", C.c_int32)]


_PD = C.POINTER(C.c_double)
_PI64 = C.POINTER(C.c_int64)


class Profile(C.Structure):
    _fields_ = [("n_layers", C.c_int32), ("t_fp", _PD), ("t_bp", _PD), ("t_c2g", _PD), ("t_g2c", _PD),
                ("t_stage", _PD), ("t_opt_gpu", _PD), ("t_opt_cpu", _PD), ("t_async", C.c_double),
                ("slot_bytes", _PI64), ("gstate_bytes", _PI64), ("fixed_bytes", C.c_int64),
                ("s_avail", C.c_int64), ("duplex", C.c_int32), ("cpu_hard", C.c_int32),
                ("cpu_util_max", C.c_double), ("decouple", C.c_int32), ("fp_serial", C.c_int32),
                ("fill_gpu", C.c_int32), ("landing_buffers", C.c_int32)]


class SolveReport(C.Structure):
    _fields_ = [("window", C.c_int32), ("w_max_memory", C.c_int32), ("reason", C.c_int32),
                ("fp_hard_ok", C.c_int32), ("bp_hard_ok", C.c_int32), ("soft_ok", C.c_int32),
                ("eq3_min_slack_ms", C.c_double), ("eq3_ok", C.c_int32), ("eq4_lhs_ms", C.c_double),
                ("eq4_rhs_ms", C.c_double), ("cpu_total_ms", C.c_double), ("gpu_step_ms", C.c_double),
                ("ring_slots", C.c_int32)]


class Stats(C.Structure):
    _fields_ = [("step", C.c_int64), ("window", C.c_int32), ("n_slots", C.c_int32), ("host_bytes", C.c_int64),
                ("device_bytes", C.c_int64), ("h2d_bytes", C.c_int64), ("d2h_bytes", C.c_int64),
                ("h2d_copies", C.c_int64), ("d2h_copies", C.c_int64), ("stage_launches", C.c_int64),
                ("h2d_busy_ms", C.c_double), ("d2h_busy_ms", C.c_double), ("h2d_profiled_bytes", C.c_int64),
                ("d2h_profiled_bytes", C.c_int64), ("cpu_adam_ms", C.c_double), ("cpu_adam_elems", C.c_int64),
                ("cpu_wait_ms", C.c_double), ("k2_ms_last", C.c_double), ("k2_bytes_last", C.c_int64),
                ("k2_launches_last", C.c_int32), ("cpu_threads", C.c_int32), ("profiled_steps", C.c_int32),
                ("k2_ms_sum", C.c_double), ("k2_bytes_sum", C.c_int64), ("k2_samples", C.c_int64),
                ("k3_ms_sum", C.c_double), ("k3_bytes_sum", C.c_int64), ("k3_samples", C.c_int64),
                ("h2d_overlap_frac", C.c_double), ("d2h_overlap_frac", C.c_double), ("last_step_ms", C.c_double),
                ("spill_bytes", C.c_int64), ("spilled_layers", C.c_int32), ("landing_buffers", C.c_int32),
                ("numa_nodes", C.c_int32), ("numa_policy", C.c_int32), ("numa_gpu_node", C.c_int32),
                ("numa_pinned_workers", C.c_int32), ("numa_bound_bytes", C.c_int64),
                ("compute_busy_ms", C.c_double), ("ring_bytes", C.c_int64), ("cpu_adam_shadow_elems", C.c_int64),
                ("shadow_layers", C.c_int32), ("spill_direct", C.c_int32), ("spill_read_bytes", C.c_int64),
                ("spill_write_bytes", C.c_int64), ("spill_io_ms", C.c_double), ("spill_uring", C.c_int32),
                ("hybrid_layers", C.c_int32), ("hybrid_updates", C.c_int64), ("hybrid_h2d_bytes", C.c_int64),
                ("hybrid_d2h_bytes", C.c_int64)]


class TraceEvent(C.Structure):
    _fields_ = [("kind", C.c_int32), ("layer", C.c_int32), ("start_ms", C.c_double), ("end_ms", C.c_double)]


TRACE_KINDS = ("fp", "bp", "h2d_fp", "h2d_bp", "d2h_grad", "k1_stage", "k3_sumsq", "k2_adamw", "cpu_adam",
               "h2d_wait_cpu")


class AdamScalars(C.Structure):
    _fields_ = [(n, C.c_float) for n in ("beta1", "beta2", "omb1", "omb2", "eps", "step_size", "sqrt_bc2", "decay")]


_lib = None


def lib() -> C.CDLL:
    """Load libsh.so (built in-tree by __graft_entry__.build()); raise loudly if absent."""
    global _lib
    if _lib is None:
        path = os.path.join(LIBDIR, "libsh.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} is missing: run `python -c 'import __graft_entry__ as g; g.build()'`")
        L = C.CDLL(path)
        vp, i32, i64, f32 = C.c_void_p, C.c_int32, C.c_int64, C.c_float
        sig = {
            "sh_init": [C.POINTER(Config), C.POINTER(vp)],
            "sh_register_host_store": [vp, i32, vp, vp, vp, i64],
            "sh_synchronize": [vp], "sh_destroy": [vp],
            "sh_forward_layer": [vp, i32, i32, vp],
            "sh_backward_layer": [vp, i32, i32, vp, vp],
            "sh_resident": [vp, vp, vp], "sh_set_lr": [vp, C.c_double],
            "sh_step": [vp, C.POINTER(C.c_double)],
            "sh_solve_window": [C.POINTER(Profile), C.POINTER(SolveReport)],
            "sh_autotune_window": [vp, C.POINTER(Profile), C.POINTER(i32)],
            "sh_set_window": [vp, i32], "sh_get_profile": [vp, C.POINTER(Profile)],
            "sh_read_layer": [vp, i32, i32, vp], "sh_stats": [vp, C.POINTER(Stats)],
            "sh_nccl_get_unique_id": [vp],
            "sh_adam_scalars_for": [C.c_double] * 5 + [i64, C.POINTER(AdamScalars)],
            "sh_op_adamw_gpu": [vp, vp, vp, vp, vp, vp, i64, i64, C.POINTER(AdamScalars), vp, vp],
            "sh_op_adamw_cpu": [vp, vp, vp, vp, vp, i64, i64, C.POINTER(AdamScalars), i32, f32, i32],
            "sh_op_cast_bf16_gpu": [vp, vp, i64, vp], "sh_op_cast_bf16_cpu": [vp, vp, i64],
            "sh_op_sumsq_gpu": [vp, i64, vp, vp],
            "sh_get_trace": [vp, vp, i32, C.POINTER(i32)],
            "sh_forward_only_end": [vp], "sh_set_window_ring": [vp, i32, i32],
            "sh_executor_grads": [vp, i32, i32, vp],
            "sh_op_exec_reduce_gpu": [vp, vp, i32, i64, f32, vp],
            "sh_numa_topology": [vp, vp, i32], "sh_numa_plan": [i32] * 5,
            "sh_numa_worker_node": [i32] * 4, "sh_numa_node_of_pci": [C.c_char_p],
            "sh_numa_bind_check": [i32, i64],
            "sh_spill_probe": [C.c_char_p, i64, C.POINTER(C.c_double), C.POINTER(C.c_double), C.POINTER(i32)],
            "sh_op_master_split_cpu": [vp, vp, vp, i64], "sh_op_master_join_cpu": [vp, vp, vp, i64],
            "sh_op_adamw_split_cpu": [vp, vp, vp, vp, vp, i64, i64, vp, i32, f32, i32],
            "sh_op_adamw_split_gpu": [vp, vp, vp, vp, vp, i64, i64, vp, vp],
        }
        for name, args in sig.items():
            fn = getattr(L, name)
            fn.argtypes = args
            fn.restype = C.c_int
        L.sh_last_error.restype = C.c_char_p
        L.sh_last_error.argtypes = []
        L.sh_abi_version.restype = C.c_int32
        L.sh_kernel_launches.restype = C.c_int64
        _lib = L
    return _lib


def check(status: int):
    if status != SH_OK:
        raise ShError(status, lib().sh_last_error().decode(errors="replace"))


def _ptr(x) -> int | None:
    """Device/host address of a torch tensor, numpy array or int (None passes NULL)."""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    if isinstance(x, np.ndarray):
        return x.ctypes.data
    raise TypeError(type(x))


def _stream_handle(stream) -> int:
    if stream is None:
        return 0
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


# ------------------------------------------------------------------------------ op level

def adam_scalars(lr, beta1, beta2, eps, weight_decay, t) -> AdamScalars:
    s = AdamScalars()
    check(lib().sh_adam_scalars_for(lr, beta1, beta2, eps, weight_decay, t, C.byref(s)))
    return s


def op_adamw_gpu(p, m, v, g, out16, out32, n, n_decay, sc: AdamScalars, coef=None, stream=None):
    check(lib().sh_op_adamw_gpu(_ptr(p), _ptr(m), _ptr(v), _ptr(g), _ptr(out16), _ptr(out32), n, n_decay,
                                C.byref(sc), _ptr(coef), _stream_handle(stream)))


def op_adamw_cpu(p, m, v, g, out16, n, n_decay, sc: AdamScalars, coef=None, threads=0):
    check(lib().sh_op_adamw_cpu(_ptr(p), _ptr(m), _ptr(v), _ptr(g), _ptr(out16), n, n_decay, C.byref(sc),
                                0 if coef is None else 1, 1.0 if coef is None else float(coef), threads))


def op_master_split_cpu(p, hi, lo, n):
    check(lib().sh_op_master_split_cpu(_ptr(p), _ptr(hi), _ptr(lo), n))


def op_master_join_cpu(hi, lo, p, n):
    check(lib().sh_op_master_join_cpu(_ptr(hi), _ptr(lo), _ptr(p), n))


def op_adamw_split_gpu(hi, lo, m, v, g, n, n_decay, sc: AdamScalars, stream=None):
    check(lib().sh_op_adamw_split_gpu(_ptr(hi), _ptr(lo), _ptr(m), _ptr(v), _ptr(g), n, n_decay, C.byref(sc),
                                      _stream_handle(stream)))


def op_adamw_split_cpu(hi, lo, m, v, g, n, n_decay, sc: AdamScalars, coef=None, threads=0):
    check(lib().sh_op_adamw_split_cpu(_ptr(hi), _ptr(lo), _ptr(m), _ptr(v), _ptr(g), n, n_decay, C.byref(sc),
                                      0 if coef is None else 1, 1.0 if coef is None else float(coef), threads))


def op_cast_bf16_gpu(src, dst16, n, stream=None):
    check(lib().sh_op_cast_bf16_gpu(_ptr(src), _ptr(dst16), n, _stream_handle(stream)))


def op_cast_bf16_cpu(src, dst16, n):
    check(lib().sh_op_cast_bf16_cpu(_ptr(src), _ptr(dst16), n))


def op_exec_reduce_gpu(dst, srcs, n, inv_k, stream=None):
    arr = (C.c_void_p * max(1, len(srcs)))(*[_ptr(x) for x in srcs])
    check(lib().sh_op_exec_reduce_gpu(_ptr(dst), arr, len(srcs), n, inv_k, _stream_handle(stream)))


def op_sumsq_gpu(g, n, out_dev, stream=None):
    check(lib().sh_op_sumsq_gpu(_ptr(g), n, _ptr(out_dev), _stream_handle(stream)))


def spill_probe(directory: str, nbytes: int = 1 << 30) -> dict:
    """NEXT-2 disk probe: O_DIRECT io_uring write / read GB/s of a fresh file in `directory`."""
    r, w, d = C.c_double(), C.c_double(), C.c_int32()
    check(lib().sh_spill_probe(directory.encode(), nbytes, C.byref(r), C.byref(w), C.byref(d)))
    return {"read_gbs": r.value, "write_gbs": w.value, "direct": bool(d.value)}


def numa_topology() -> list[tuple[int, int]]:
    """[(node id, cpu count)] of the online NUMA nodes (sysfs; SH_SYSFS_ROOT prefixes it)."""
    ids, cpus = (C.c_int32 * 1024)(), (C.c_int32 * 1024)()
    n = lib().sh_numa_topology(C.addressof(ids), C.addressof(cpus), 1024)
    return [(ids[k], cpus[k]) for k in range(n)]


def numa_plan(policy: int, unit: int, n_nodes: int, gpu_node: int = 0, shared: bool = False) -> int:
    return lib().sh_numa_plan(policy, unit, n_nodes, gpu_node, int(shared))


def numa_worker_node(policy: int, tid: int, n_threads: int, gpu_node: int = 0) -> int:
    return lib().sh_numa_worker_node(policy, tid, n_threads, gpu_node)


def numa_node_of_pci(bus_id: str) -> int:
    return lib().sh_numa_node_of_pci(bus_id.encode())


def numa_bind_check(node_id: int, nbytes: int) -> int:
    return lib().sh_numa_bind_check(node_id, nbytes)


def kernel_launches() -> int:
    return int(lib().sh_kernel_launches())


def nccl_unique_id() -> bytes:
    buf = (C.c_uint8 * 128)()
    check(lib().sh_nccl_get_unique_id(buf))
    return bytes(buf)


# ------------------------------------------------------------------------------ solver

def _dbl(a, n):
    if a is None:
        return None
    arr = np.ascontiguousarray(np.asarray(a, dtype=np.float64).reshape(n))
    return arr


def make_profile(t_fp, t_bp, t_c2g, t_g2c, t_stage=None, t_opt_gpu=None, t_opt_cpu=None, t_async=0.0,
                 slot_bytes=None, gstate_bytes=None, fixed_bytes=0, s_avail=2 ** 62, duplex=False,
                 cpu_hard=False, cpu_util_max=1.0, decouple=False, fp_serial=False, fill_gpu=False,
                 landing_buffers=0):
    """(Profile, keep-alive arrays) for sh_solve_window / sh_autotune_window."""
    n = len(t_fp)
    keep = {}
    prof = Profile()
    prof.n_layers = n
    for name, a in (("t_fp", t_fp), ("t_bp", t_bp), ("t_c2g", t_c2g), ("t_g2c", t_g2c), ("t_stage", t_stage),
                    ("t_opt_gpu", t_opt_gpu), ("t_opt_cpu", t_opt_cpu)):
        arr = _dbl(a, n)
        keep[name] = arr
        setattr(prof, name, arr.ctypes.data_as(_PD) if arr is not None else None)
    for name, a in (("slot_bytes", slot_bytes), ("gstate_bytes", gstate_bytes)):
        arr = None if a is None else np.ascontiguousarray(np.asarray(a, dtype=np.int64).reshape(n))
        keep[name] = arr
        setattr(prof, name, arr.ctypes.data_as(_PI64) if arr is not None else None)
    prof.t_async = t_async
    prof.fixed_bytes = int(fixed_bytes)
    prof.s_avail = int(s_avail)
    prof.duplex = 1 if duplex else 0
    prof.cpu_hard = 1 if cpu_hard else 0
    prof.cpu_util_max = cpu_util_max
    prof.decouple = 1 if decouple else 0
    prof.fp_serial = 1 if fp_serial else 0
    prof.fill_gpu = 1 if fill_gpu else 0
    prof.landing_buffers = int(landing_buffers)
    return prof, keep


def solve_window(*args, **kw) -> dict:
    """Pure call of sh_solve_window (no GPU); arguments as make_profile."""
    prof, _keep = make_profile(*args, **kw)
    rep = SolveReport()
    check(lib().sh_solve_window(C.byref(prof), C.byref(rep)))
    return {f: getattr(rep, f) for f, _ in SolveReport._fields_}


# ------------------------------------------------------------------------------ engine

class Engine:
    """One STRONGHOLD engine context (one per GPU / rank)."""

    def __init__(self, layer_numels, layer_wd, res_numels, res_wd, *, window, precision=SH_BF16_MIXED,
                 lr=1.5e-4, betas=(0.9, 0.999), eps=1e-8, weight_decay=0.01, max_grad_norm=0.0, device=0,
                 stream=None, cpu_threads=0, grad_ring_depth=0, warmup_steps=5, device_budget_bytes=0,
                 world_size=1, rank=0, nccl_id: bytes | None = None, flags=0, shm_name: str | None = None,
                 ring_slots=0, cpu_util_max=0.0, n_executors=1, spill_dir: str | None = None,
                 host_pin_budget_bytes=0, warmup_window=0, numa_policy=0, ring_bytes=0, hybrid_layers=0):
        L = lib()
        self.n_layers = len(layer_numels)
        self._keep = []
        shapes = (LayerShape * self.n_layers)()
        self.layer_numels = [list(map(int, n)) for n in layer_numels]
        for i, (nums, wds) in enumerate(zip(layer_numels, layer_wd)):
            shapes[i] = self._shape(nums, wds)
        cfg = Config()
        cfg.n_layers = self.n_layers
        cfg.layers = shapes
        cfg.resident = self._shape(res_numels, res_wd)
        self.res_numels = list(map(int, res_numels))
        cfg.window = window
        cfg.precision = precision
        cfg.lr = lr
        cfg.beta1, cfg.beta2 = betas
        cfg.eps = eps
        cfg.weight_decay = weight_decay
        cfg.max_grad_norm = max_grad_norm
        cfg.device = device
        cfg.compute_stream = _stream_handle(stream)
        cfg.cpu_threads = cpu_threads
        cfg.grad_ring_depth = grad_ring_depth
        cfg.warmup_steps = warmup_steps
        cfg.device_budget_bytes = device_budget_bytes
        cfg.ring_slots = ring_slots
        cfg.cpu_util_max = cpu_util_max
        cfg.world_size = world_size
        cfg.rank = rank
        idbuf = None
        if nccl_id is not None:
            idbuf = (C.c_uint8 * 128).from_buffer_copy(nccl_id)
            cfg.nccl_unique_id = C.cast(idbuf, C.c_void_p)
        cfg.flags = flags
        cfg.n_executors = n_executors
        self._spill = spill_dir.encode() if spill_dir else None
        cfg.spill_dir = self._spill
        cfg.host_pin_budget_bytes = int(host_pin_budget_bytes)
        cfg.warmup_window = int(warmup_window)
        cfg.numa_policy = int(numa_policy)
        cfg.ring_bytes = int(ring_bytes)
        cfg.hybrid_layers = int(hybrid_layers)
        self.n_executors = max(1, n_executors)
        self._shm = shm_name.encode() if shm_name else None
        cfg.shm_name = self._shm
        self.precision = precision
        self._cfg = cfg
        self._shapes = shapes
        h = C.c_void_p()
        check(L.sh_init(C.byref(cfg), C.byref(h)))
        self.h = h
        self._p_arr = [(C.c_void_p * len(n))() for n in self.layer_numels]
        self._g_arr = [(C.c_void_p * len(n))() for n in self.layer_numels]
        self._rp = (C.c_void_p * len(res_numels))()
        self._rg = (C.c_void_p * len(res_numels))()
        check(L.sh_resident(self.h, self._rp, self._rg))
        # executor e >= 1 gradient pointer arrays: per layer (filled at each backward PRE) and resident
        self._xg = [[(C.c_void_p * len(n))() for n in self.layer_numels] for _ in range(self.n_executors)]
        self._xr = [(C.c_void_p * len(res_numels))() for _ in range(self.n_executors)]
        for e in range(1, self.n_executors):
            check(L.sh_executor_grads(self.h, -1, e, self._xr[e]))
        self._L = L

    def _shape(self, nums, wds):
        n = np.ascontiguousarray(np.asarray(nums, dtype=np.int64))
        w = np.ascontiguousarray(np.asarray(wds, dtype=np.uint8))
        self._keep += [n, w]
        s = LayerShape()
        s.n_tensors = len(nums)
        s.numel = n.ctypes.data_as(C.POINTER(C.c_int64))
        s.weight_decay = w.ctypes.data_as(C.POINTER(C.c_uint8))
        return s

    # -- lifecycle
    def register(self, layer: int, params: np.ndarray, m=None, v=None, step: int = 0):
        p = np.ascontiguousarray(params, dtype=np.float32)
        mm = None if m is None else np.ascontiguousarray(m, dtype=np.float32)
        vv = None if v is None else np.ascontiguousarray(v, dtype=np.float32)
        check(self._L.sh_register_host_store(self.h, layer, p.ctypes.data, None if mm is None else mm.ctypes.data,
                                             None if vv is None else vv.ctypes.data, step))

    def synchronize(self):
        check(self._L.sh_synchronize(self.h))

    def close(self):
        if getattr(self, "h", None):
            self._L.sh_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # -- hooks
    def forward_pre(self, i: int):
        a = self._p_arr[i]
        check(self._L.sh_forward_layer(self.h, i, SH_PRE, a))
        return a

    def forward_post(self, i: int):
        check(self._L.sh_forward_layer(self.h, i, SH_POST, None))

    def backward_pre(self, i: int):
        a, g = self._p_arr[i], self._g_arr[i]
        check(self._L.sh_backward_layer(self.h, i, SH_PRE, a, g))
        return a, g

    def executor_grads(self, i: int, e: int):
        """Gradient pointers of executor e for layer i (between its backward PRE and POST)."""
        if e == 0:
            return self._g_arr[i]
        g = self._xg[e][i] if 0 <= e < self.n_executors else (C.c_void_p * 64)()  # C reports the error
        check(self._L.sh_executor_grads(self.h, i, e, g))
        return g

    def executor_resident_grads(self, e: int):
        return self._rg if e == 0 else self._xr[e]

    def backward_post(self, i: int):
        check(self._L.sh_backward_layer(self.h, i, SH_POST, None, None))

    def forward_only_end(self):
        check(self._L.sh_forward_only_end(self.h))

    def resident(self):
        return self._rp, self._rg

    def set_lr(self, lr: float):
        check(self._L.sh_set_lr(self.h, lr))

    def step(self, want_norm: bool = False):
        if want_norm:
            d = C.c_double()
            check(self._L.sh_step(self.h, C.byref(d)))
            return d.value
        check(self._L.sh_step(self.h, None))
        return None

    # -- window
    def set_window(self, w: int, ring_slots: int | None = None):
        if ring_slots is None:
            check(self._L.sh_set_window(self.h, w))
        else:
            check(self._L.sh_set_window_ring(self.h, w, ring_slots))

    def autotune(self, override: dict | None = None) -> int:
        """Solve on the measured profile, or on `override` (make_profile keyword arguments), and apply."""
        w = C.c_int32()
        if override is None:
            check(self._L.sh_autotune_window(self.h, None, C.byref(w)))
        else:
            prof, _keep = make_profile(**override)
            check(self._L.sh_autotune_window(self.h, C.byref(prof), C.byref(w)))
        return w.value

    def profile(self) -> dict:
        p = Profile()
        check(self._L.sh_get_profile(self.h, C.byref(p)))
        n = p.n_layers
        out = {"n_layers": n, "t_async": p.t_async, "s_avail": p.s_avail, "fixed_bytes": p.fixed_bytes,
               "duplex": p.duplex, "cpu_hard": p.cpu_hard, "cpu_util_max": p.cpu_util_max, "decouple": p.decouple,
               "fp_serial": p.fp_serial, "fill_gpu": p.fill_gpu, "landing_buffers": p.landing_buffers}
        for f in ("t_fp", "t_bp", "t_c2g", "t_g2c", "t_stage", "t_opt_gpu", "t_opt_cpu"):
            out[f] = [getattr(p, f)[i] for i in range(n)]
        for f in ("slot_bytes", "gstate_bytes"):
            out[f] = [getattr(p, f)[i] for i in range(n)]
        return out

    # -- inspection
    def read_layer(self, layer: int, what: int = SH_READ_PARAM) -> np.ndarray:
        n = sum(self.res_numels) if layer < 0 else sum(self.layer_numels[layer])
        if what == SH_READ_COMPUTE and self.precision == SH_BF16_MIXED:
            out = np.empty(n, dtype=np.uint16)
        else:
            out = np.empty(n, dtype=np.float32)
        check(self._L.sh_read_layer(self.h, layer, what, out.ctypes.data))
        return out

    def trace(self) -> list[dict]:
        """Intervals of the last profiled step (ms from its first FP hook)."""
        n = C.c_int32()
        check(self._L.sh_get_trace(self.h, None, 0, C.byref(n)))
        buf = (TraceEvent * max(1, n.value))()
        check(self._L.sh_get_trace(self.h, buf, n.value, C.byref(n)))
        return [{"kind": TRACE_KINDS[e.kind], "layer": e.layer, "start_ms": e.start_ms, "end_ms": e.end_ms}
                for e in buf[:n.value]]

    def stats(self) -> dict:
        s = Stats()
        check(self._L.sh_stats(self.h, C.byref(s)))
        return {f: getattr(s, f) for f, _ in Stats._fields_}
