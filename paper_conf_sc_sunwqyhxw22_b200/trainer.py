"""The training loop that drives the engine: the role of the user's unmodified model code plus
the framework hooks STRONGHOLD registers.  Per layer it calls the engine's
PRE hook, the (outside-hot-path) GPT block compute on the returned slot pointers, and the POST
hook.  Marshalling only: no arithmetic happens in Python.

torch is used for device memory (token / loss buffers), the compute stream and pinned host
buffers -- plumbing, as the task's north star states.
"""
from __future__ import annotations

import math
from dataclasses import dataclass

import numpy as np
import torch

import synth

from . import sh
from .gpt import GPT, FlashAttention


@dataclass
class ModelConfig:
    n_layers: int
    hidden: int
    heads: int
    seq: int
    vocab: int

    def layer_numels(self):
        return [int(np.prod(s)) for s in synth.layer_shapes(self.hidden)]

    def res_numels(self):
        return [int(np.prod(s)) for s in synth.resident_shapes(self.vocab, self.seq, self.hidden)]

    def params_per_layer(self):
        return sum(self.layer_numels())

    def n_params(self):
        return self.n_layers * self.params_per_layer() + sum(self.res_numels())

    def flops_per_token(self):
        """Model flops per token of one training step with layer-wise recompute: layers do
        fwd + recompute + bwd = 4 fwd units (8 flop/param), the tied head fwd + bwd (6 h V);
        causal attention scores / values are reported separately."""
        return 8 * self.n_layers * self.params_per_layer() + 6 * self.hidden * self.vocab


class StrongholdTrainer:
    """GPT-2 training with the working-window engine on one GPU (one rank)."""

    def __init__(self, mc: ModelConfig, *, batch: int, window: int, precision=sh.SH_BF16_MIXED, lr=1.5e-4,
                 max_grad_norm=0.0, device=0, seed=1234, cpu_threads=0, grad_ring_depth=0, warmup_steps=5,
                 flags=0, world_size=1, rank=0, nccl_id=None, init=True, init_threads=8, shm_name=None,
                 attention="auto", ring_slots=0):
        self.mc = mc
        self.batch = batch
        self.device = torch.device("cuda", device)
        torch.cuda.set_device(self.device)
        self.stream = torch.cuda.Stream(device=self.device)
        L = mc.n_layers
        self.engine = sh.Engine([mc.layer_numels()] * L, [synth.layer_weight_decay(mc.hidden)] * L,
                                mc.res_numels(), synth.resident_weight_decay(), window=window,
                                precision=precision, lr=lr, max_grad_norm=max_grad_norm, device=device,
                                stream=self.stream, cpu_threads=cpu_threads, grad_ring_depth=grad_ring_depth,
                                warmup_steps=warmup_steps, world_size=world_size, rank=rank, nccl_id=nccl_id,
                                flags=flags, shm_name=shm_name, ring_slots=ring_slots)
        self.gpt = GPT(n_layers=L, hidden=mc.hidden, heads=mc.heads, seq=mc.seq, max_batch=batch,
                       vocab=mc.vocab, precision=precision, device=device, stream=self.stream)
        # attention core: fused flash-attention library kernel on the bf16 path ("auto"/"flash"),
        # else the cuBLAS batched-GEMM + softmax kernels inside libsh_gpt ("cublas", and fp32 mode)
        self.flash = None
        if attention == "flash" or (attention == "auto" and precision == sh.SH_BF16_MIXED):
            try:
                self.flash = FlashAttention(self.gpt, batch, mc.seq, mc.hidden, mc.heads)
            except ImportError:
                if attention == "flash":
                    raise
        self.tok_dev = torch.empty((batch, mc.seq + 1), dtype=torch.int32, device=self.device)
        self.loss_dev = torch.zeros(1, dtype=torch.float32, device=self.device)
        self.loss_host = torch.zeros(1, dtype=torch.float32).pin_memory()
        # with a shared host store only rank 0 writes the host-optimised layers' initial state
        self._w0 = window if window >= 0 else min(2, L)
        self._host_data_skipped = bool(shm_name) and rank != 0
        if init:
            self.init_params(seed, init_threads)

    def init_params(self, seed: int, threads: int = 8):
        """Seeded init (synth/, bit-identical to synth.init_layer) streamed layer by layer through
        one reusable buffer: O(one layer) of transient host memory at any model size."""
        mc = self.mc
        flat = np.empty(mc.params_per_layer(), np.float32)
        for i in range(mc.n_layers):
            if self._host_data_skipped and i >= self._w0:
                flat[:] = 0.0  # ignored by the engine: rank 0 writes the shared copy
            else:
                synth.init_layer_into(flat, seed, i, mc.n_layers, mc.hidden, threads)
            self.engine.register(i, flat)
        res = np.empty(sum(mc.res_numels()), np.float32)
        synth.init_resident_into(res, seed, mc.vocab, mc.seq, mc.hidden, threads)
        self.engine.register(-1, res)

    def register_state(self, layers, resident, m_layers=None, v_layers=None, m_res=None, v_res=None, step=0):
        flat = lambda ts: np.concatenate([np.asarray(a, np.float32).reshape(-1) for a in ts])
        for i, P in enumerate(layers):
            self.engine.register(i, flat(P), None if m_layers is None else flat(m_layers[i]),
                                 None if v_layers is None else flat(v_layers[i]), step)
        self.engine.register(-1, flat(resident), None if m_res is None else flat(m_res),
                             None if v_res is None else flat(v_res), step)

    # ------------------------------------------------------------------ one step
    def step_device(self, batch: int | None = None, want_norm=False):
        """One training step on tokens already in self.tok_dev.  Asynchronous unless want_norm."""
        e, g = self.engine, self.gpt
        B = batch or self.batch
        tok = self.tok_dev.data_ptr()
        rp, rg = e.resident()
        L = self.mc.n_layers
        fa = self.flash
        if fa is not None:
            fa.set_batch(B)
        with torch.cuda.stream(self.stream):
            # FP: pre_forward -> compute -> post_forward
            for i in range(L):
                P = e.forward_pre(i)
                if i == 0:
                    g.embed_forward(tok, B, rp)
                if fa is None:
                    g.layer_forward(i, P)
                else:
                    g.forward_qkv(i, P)
                    fa.forward()
                    g.forward_out(i, P, True)
                e.forward_post(i)
            g.head(tok, rp, rg, self.loss_dev.data_ptr())
            # BP: pre_backward -> recompute + backward -> post (offload + CPU Adam)
            for i in range(L - 1, -1, -1):
                P, G = e.backward_pre(i)
                if fa is None:
                    g.layer_backward(i, P, G)
                else:
                    g.forward_qkv(i, P)       # recompute from the layer's checkpoint
                    fa.forward()
                    g.forward_out(i, P, False)
                    g.backward_mlp(i, P, G)
                    fa.backward()
                    g.backward_qkv(i, P, G)
                e.backward_post(i)
            g.embed_backward(tok, rg)
            return e.step(want_norm=want_norm)

    def forward_only(self, batch: int | None = None) -> None:
        """FP-only pass (streaming inference / KD teacher) over self.tok_dev:
        loss -> self.loss_dev; no backward, no update (NEXT-4)."""
        e, g = self.engine, self.gpt
        B = batch or self.batch
        tok = self.tok_dev.data_ptr()
        rp, _ = e.resident()
        fa = self.flash
        if fa is not None:
            fa.set_batch(B)
        with torch.cuda.stream(self.stream):
            for i in range(self.mc.n_layers):
                P = e.forward_pre(i)
                if i == 0:
                    g.embed_forward(tok, B, rp)
                if fa is None:
                    g.layer_forward(i, P)
                else:
                    g.forward_qkv(i, P)
                    fa.forward()
                    g.forward_out(i, P, True)
                e.forward_post(i)
            g.head_forward(tok, rp, self.loss_dev.data_ptr())
            e.forward_only_end()

    def step(self, tokens_host: torch.Tensor, want_norm=False) -> float:
        """End-to-end public step: pinned host tokens -> device, train, loss -> host."""
        with torch.cuda.stream(self.stream):
            self.tok_dev[: tokens_host.shape[0]].copy_(tokens_host, non_blocking=True)
        self.step_device(tokens_host.shape[0], want_norm)
        with torch.cuda.stream(self.stream):
            self.loss_host.copy_(self.loss_dev, non_blocking=True)
        self.stream.synchronize()
        return float(self.loss_host.item())

    def set_tokens(self, tokens: np.ndarray):
        t = torch.from_numpy(np.ascontiguousarray(tokens, dtype=np.int32))
        with torch.cuda.stream(self.stream):
            self.tok_dev[: t.shape[0]].copy_(t.to(self.device), non_blocking=False)
        self.stream.synchronize()

    def loss(self) -> float:
        self.stream.synchronize()
        return float(self.loss_dev.item())

    # ------------------------------------------------------------------ state
    def read_layer_tensors(self, layer: int, what=sh.SH_READ_PARAM):
        flat = self.engine.read_layer(layer, what)
        shapes = synth.layer_shapes(self.mc.hidden) if layer >= 0 else \
            synth.resident_shapes(self.mc.vocab, self.mc.seq, self.mc.hidden)
        out, o = [], 0
        for s in shapes:
            n = int(np.prod(s))
            out.append(flat[o:o + n].reshape(s))
            o += n
        return out

    def close(self):
        self.engine.close()
        self.gpt.close()


def bf16_bits_to_f32(u16: np.ndarray) -> np.ndarray:
    return (u16.astype(np.uint32) << 16).view(np.float32)
