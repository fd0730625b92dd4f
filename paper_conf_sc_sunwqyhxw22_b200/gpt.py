"""ctypes binding of libsh_gpt.so (include/sh_gpt.h) -- the GPT block compute that drives the
engine.  OUTSIDE THE HOT PATH (labelled per BASELINE.json north_star); marshalling only."""
from __future__ import annotations

import ctypes as C
import os

from .sh import LIBDIR

EXPORTS = ("gpt_create", "gpt_destroy", "gpt_last_error", "gpt_workspace_bytes", "gpt_embed_forward",
           "gpt_layer_forward", "gpt_head_forward_backward", "gpt_layer_backward", "gpt_embed_backward",
           "gpt_checkpoint", "gpt_kernel_launches", "gpt_layer_forward_qkv", "gpt_layer_forward_out",
           "gpt_layer_backward_mlp", "gpt_layer_backward_qkv", "gpt_buffer", "gpt_head_forward")


class GptConfig(C.Structure):
    _fields_ = [("n_layers", C.c_int32), ("hidden", C.c_int32), ("heads", C.c_int32), ("seq", C.c_int32),
                ("max_batch", C.c_int32), ("vocab", C.c_int32), ("precision", C.c_int32), ("device", C.c_int32),
                ("stream", C.c_void_p)]


_lib = None


def lib() -> C.CDLL:
    global _lib
    if _lib is None:
        path = os.path.join(LIBDIR, "libsh_gpt.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} is missing: run __graft_entry__.build()")
        L = C.CDLL(path)
        vp, i32 = C.c_void_p, C.c_int32
        sig = {"gpt_create": [C.POINTER(GptConfig), C.POINTER(vp)], "gpt_destroy": [vp],
               "gpt_embed_forward": [vp, vp, i32, vp], "gpt_layer_forward": [vp, i32, vp],
               "gpt_head_forward_backward": [vp, vp, vp, vp, vp], "gpt_layer_backward": [vp, i32, vp, vp],
               "gpt_embed_backward": [vp, vp, vp], "gpt_layer_forward_qkv": [vp, i32, vp],
               "gpt_layer_forward_out": [vp, i32, vp, i32], "gpt_layer_backward_mlp": [vp, i32, vp, vp],
               "gpt_layer_backward_qkv": [vp, i32, vp, vp], "gpt_head_forward": [vp, vp, vp, vp]}
        for n, a in sig.items():
            getattr(L, n).argtypes = a
            getattr(L, n).restype = C.c_int32
        L.gpt_last_error.restype = C.c_char_p
        L.gpt_workspace_bytes.argtypes = [vp]
        L.gpt_workspace_bytes.restype = C.c_int64
        L.gpt_checkpoint.argtypes = [vp, i32]
        L.gpt_checkpoint.restype = C.c_void_p
        L.gpt_kernel_launches.restype = C.c_int64
        L.gpt_buffer.argtypes = [vp, i32]
        L.gpt_buffer.restype = C.c_void_p
        _lib = L
    return _lib


def kernel_launches() -> int:
    return int(lib().gpt_kernel_launches())


def _check(r):
    if r != 0:
        raise RuntimeError(f"gpt status {r}: {lib().gpt_last_error().decode(errors='replace')}")


class GPT:
    def __init__(self, *, n_layers, hidden, heads, seq, max_batch, vocab, precision, device=0, stream=None):
        cfg = GptConfig(n_layers, hidden, heads, seq, max_batch, vocab, precision, device,
                        stream if isinstance(stream, int) else stream.cuda_stream)
        h = C.c_void_p()
        _check(lib().gpt_create(C.byref(cfg), C.byref(h)))
        self.h = h
        self._L = lib()

    def workspace_bytes(self) -> int:
        return self._L.gpt_workspace_bytes(self.h)

    def embed_forward(self, tok_ptr: int, batch: int, res_params):
        _check(self._L.gpt_embed_forward(self.h, tok_ptr, batch, res_params))

    def layer_forward(self, layer: int, params):
        _check(self._L.gpt_layer_forward(self.h, layer, params))

    def head(self, tok_ptr: int, res_params, res_grads, loss_ptr: int):
        _check(self._L.gpt_head_forward_backward(self.h, tok_ptr, res_params, res_grads, loss_ptr))

    def head_forward(self, tok_ptr: int, res_params, loss_ptr: int):
        _check(self._L.gpt_head_forward(self.h, tok_ptr, res_params, loss_ptr))

    def layer_backward(self, layer: int, params, grads):
        _check(self._L.gpt_layer_backward(self.h, layer, params, grads))

    def embed_backward(self, tok_ptr: int, res_grads):
        _check(self._L.gpt_embed_backward(self.h, tok_ptr, res_grads))

    # staged block (attention core supplied by the caller)
    def forward_qkv(self, layer, params):
        _check(self._L.gpt_layer_forward_qkv(self.h, layer, params))

    def forward_out(self, layer, params, write_out=True):
        _check(self._L.gpt_layer_forward_out(self.h, layer, params, 1 if write_out else 0))

    def backward_mlp(self, layer, params, grads):
        _check(self._L.gpt_layer_backward_mlp(self.h, layer, params, grads))

    def backward_qkv(self, layer, params, grads):
        _check(self._L.gpt_layer_backward_qkv(self.h, layer, params, grads))

    def buffer_ptr(self, which: int) -> int:
        return self._L.gpt_buffer(self.h, which)

    def checkpoint_ptr(self, layer: int) -> int:
        return self._L.gpt_checkpoint(self.h, layer)

    def close(self):
        if getattr(self, "h", None):
            self._L.gpt_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class _CudaArray:
    """Minimal __cuda_array_interface__ view of a device pointer (for torch.as_tensor)."""

    def __init__(self, ptr: int, n: int, typestr: str):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False), "version": 3,
                                         "strides": None, "stream": None}


class FlashAttention:
    """Causal attention core of the bf16 path through the flash_attn 2.8 library kernels (sm_100
    SASS; library code like cuBLAS, OUTSIDE the hot path): the S x S scores are never materialised.
    Backward runs with deterministic=True so gradients are bit-reproducible (the engine's
    bit-exact-across-window property needs a deterministic driver)."""

    def __init__(self, gpt: "GPT", max_batch: int, seq: int, hidden: int, heads: int):
        import torch
        import flash_attn_2_cuda as fa  # noqa: F401  (fails loudly if the library is absent)
        self.fa = fa
        self.S, self.h, self.nh, self.hd = seq, hidden, heads, hidden // heads
        self.scale = 1.0 / (self.hd ** 0.5)
        n = max_batch * seq
        def wrap(which, cols):
            t = torch.as_tensor(_CudaArray(gpt.buffer_ptr(which), n * cols, "<i2"), device="cuda")
            return t.view(torch.bfloat16)
        self._qkv, self._att = wrap(0, 3 * hidden), wrap(1, hidden)
        self._datt, self._dqkv = wrap(2, hidden), wrap(3, 3 * hidden)
        self.lse = self.rng = None
        self.B = None

    def set_batch(self, B: int):
        if B == self.B:
            return
        S, nh, hd = self.S, self.nh, self.hd
        n = B * S
        qkv = self._qkv[: n * 3 * self.h].view(B, S, 3, nh, hd)
        dqkv = self._dqkv[: n * 3 * self.h].view(B, S, 3, nh, hd)
        self.q, self.k, self.v = qkv[:, :, 0], qkv[:, :, 1], qkv[:, :, 2]
        self.dq, self.dk, self.dv = dqkv[:, :, 0], dqkv[:, :, 1], dqkv[:, :, 2]
        self.att = self._att[: n * self.h].view(B, S, nh, hd)
        self.datt = self._datt[: n * self.h].view(B, S, nh, hd)
        self.B = B

    def forward(self):
        _, self.lse, _, self.rng = self.fa.fwd(self.q, self.k, self.v, self.att, None, 0.0, self.scale, True,
                                               -1, -1, 0.0, False, None)

    def backward(self):
        self.fa.bwd(self.datt, self.q, self.k, self.v, self.att, self.lse, self.dq, self.dk, self.dv, None, 0.0,
                    self.scale, True, -1, -1, 0.0, True, None, self.rng)
