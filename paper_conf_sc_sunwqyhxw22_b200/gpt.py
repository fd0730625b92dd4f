"""ctypes binding of libsh_gpt.so (include/sh_gpt.h) -- the GPT block compute that drives the
engine.  OUTSIDE THE HOT PATH (labelled per BASELINE.json north_star); marshalling only."""
from __future__ import annotations

import ctypes as C
import os

from .sh import LIBDIR

EXPORTS = ("gpt_create", "gpt_destroy", "gpt_last_error", "gpt_workspace_bytes", "gpt_embed_forward",
           "gpt_layer_forward", "gpt_head_forward_backward", "gpt_layer_backward", "gpt_embed_backward",
           "gpt_checkpoint", "gpt_kernel_launches")


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
               "gpt_embed_backward": [vp, vp, vp]}
        for n, a in sig.items():
            getattr(L, n).argtypes = a
            getattr(L, n).restype = C.c_int32
        L.gpt_last_error.restype = C.c_char_p
        L.gpt_workspace_bytes.argtypes = [vp]
        L.gpt_workspace_bytes.restype = C.c_int64
        L.gpt_checkpoint.argtypes = [vp, i32]
        L.gpt_checkpoint.restype = C.c_void_p
        L.gpt_kernel_launches.restype = C.c_int64
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

    def layer_backward(self, layer: int, params, grads):
        _check(self._L.gpt_layer_backward(self.h, layer, params, grads))

    def embed_backward(self, tok_ptr: int, res_grads):
        _check(self._L.gpt_embed_backward(self.h, tok_ptr, res_grads))

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
