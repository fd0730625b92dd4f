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
                 attention="auto", ring_slots=0, executors=1, spill_dir=None, host_pin_budget_bytes=0,
                 warmup_window=0, numa_policy=0, ring_bytes=0, hybrid_layers=0):
        self.mc = mc
        self.batch = batch
        # NEXT-3 multi-stream executors: K workers on K streams, one parameter copy,
        # each on batch/K sequences; the engine's K4 averages their gradients before the update
        self.K = max(1, int(executors))
        if batch % self.K:
            raise ValueError(f"batch {batch} is not a multiple of executors {self.K}")
        self.mb = batch // self.K
        self.device = torch.device("cuda", device)
        torch.cuda.set_device(self.device)
        self.stream = torch.cuda.Stream(device=self.device)
        L = mc.n_layers
        self.engine = sh.Engine([mc.layer_numels()] * L, [synth.layer_weight_decay(mc.hidden)] * L,
                                mc.res_numels(), synth.resident_weight_decay(), window=window,
                                precision=precision, lr=lr, max_grad_norm=max_grad_norm, device=device,
                                stream=self.stream, cpu_threads=cpu_threads, grad_ring_depth=grad_ring_depth,
                                warmup_steps=warmup_steps, world_size=world_size, rank=rank, nccl_id=nccl_id,
                                flags=flags, shm_name=shm_name, ring_slots=ring_slots, n_executors=self.K,
                                spill_dir=spill_dir, host_pin_budget_bytes=host_pin_budget_bytes,
                                warmup_window=warmup_window, numa_policy=numa_policy, ring_bytes=ring_bytes,
                                hybrid_layers=hybrid_layers)
        # executor 0 runs on the engine's compute stream, executors >= 1 on their own streams
        self.streams = [self.stream] + [torch.cuda.Stream(device=self.device) for _ in range(self.K - 1)]
        self.gpts = [GPT(n_layers=L, hidden=mc.hidden, heads=mc.heads, seq=mc.seq, max_batch=self.mb,
                         vocab=mc.vocab, precision=precision, device=device, stream=st) for st in self.streams]
        self.gpt = self.gpts[0]
        # attention core: fused flash-attention library kernel on the bf16 path ("auto"/"flash"),
        # else the cuBLAS batched-GEMM + softmax kernels inside libsh_gpt ("cublas", and fp32 mode)
        self.flashes = [None] * self.K
        if attention == "flash" or (attention == "auto" and precision == sh.SH_BF16_MIXED):
            try:
                self.flashes = [FlashAttention(g, self.mb, mc.seq, mc.hidden, mc.heads) for g in self.gpts]
            except ImportError:
                if attention == "flash":
                    raise
        self.flash = self.flashes[0]
        self._fork = [torch.cuda.Event() for _ in range(2 * mc.n_layers + 2)]
        self._join = [[torch.cuda.Event() for _ in range(2 * mc.n_layers + 2)] for _ in range(self.K)]
        self.tok_dev = torch.empty((batch, mc.seq + 1), dtype=torch.int32, device=self.device)
        self.loss_dev = torch.zeros(1, dtype=torch.float32, device=self.device)
        self.loss_parts = torch.zeros(self.K, dtype=torch.float32, device=self.device)
        self.loss_host = torch.zeros(1, dtype=torch.float32).pin_memory()
        # with a shared host store only rank 0 writes the host-optimised layers' initial state
        self._w0 = window if window >= 0 else min(warmup_window if warmup_window > 0 else 2, L)
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
    def _run(self, k: int, fn):
        """Run fn(e) for every executor e: executor 0 on the compute stream, executors >= 1 forked
        from the compute stream's current position (after the hook just issued) on their own
        streams and joined back before the next hook (the sh_executor_grads contract)."""
        if self.K == 1:
            fn(0)
            return
        cs = self.stream
        self._fork[k].record(cs)
        for e in range(1, self.K):
            st = self.streams[e]
            st.wait_event(self._fork[k])
            with torch.cuda.stream(st):
                fn(e)
            self._join[e][k].record(st)
        fn(0)
        for e in range(1, self.K):
            cs.wait_event(self._join[e][k])

    def _tok(self, e: int, mb: int) -> int:
        return self.tok_dev.data_ptr() + 4 * e * mb * (self.mc.seq + 1)

    def _layer_fwd(self, e: int, i: int, P, write_out=True):
        g, fa = self.gpts[e], self.flashes[e]
        if fa is None:
            if write_out:
                g.layer_forward(i, P)
            else:
                raise AssertionError("recompute without flash goes through layer_backward")
        else:
            g.forward_qkv(i, P)
            fa.forward()
            g.forward_out(i, P, write_out)

    def step_device(self, batch: int | None = None, want_norm=False):
        """One training step on tokens already in self.tok_dev.  Asynchronous unless want_norm."""
        e = self.engine
        B = batch or self.batch
        if B % self.K:
            raise ValueError(f"batch {B} is not a multiple of executors {self.K}")
        mb = B // self.K
        L = self.mc.n_layers
        for fa in self.flashes:
            if fa is not None:
                fa.set_batch(mb)
        gp = self.gpts
        loss = [self.loss_dev.data_ptr()] if self.K == 1 else \
            [self.loss_parts.data_ptr() + 4 * x for x in range(self.K)]
        with torch.cuda.stream(self.stream):
            # FP: pre_forward -> compute -> post_forward
            for i in range(L):
                P = e.forward_pre(i)

                def fwd(x, i=i, P=P):
                    if i == 0:
                        gp[x].embed_forward(self._tok(x, mb), mb, e.resident()[0])
                    self._layer_fwd(x, i, P)
                self._run(i, fwd)
                e.forward_post(i)
            rp = e.resident()[0]
            self._run(L, lambda x: gp[x].head(self._tok(x, mb), rp, e.executor_resident_grads(x), loss[x]))
            # BP: pre_backward -> recompute + backward -> post (offload + CPU Adam)
            for i in range(L - 1, -1, -1):
                P, _ = e.backward_pre(i)
                Gs = [e.executor_grads(i, x) for x in range(self.K)]

                def bwd(x, i=i, P=P):
                    g, fa, G = gp[x], self.flashes[x], Gs[x]
                    if fa is None:
                        g.layer_backward(i, P, G)
                    else:
                        g.forward_qkv(i, P)       # recompute from the layer's checkpoint
                        fa.forward()
                        g.forward_out(i, P, False)
                        g.backward_mlp(i, P, G)
                        fa.backward()
                        g.backward_qkv(i, P, G)
                self._run(L + 1 + (L - 1 - i), bwd)
                e.backward_post(i)
            self._run(2 * L + 1, lambda x: gp[x].embed_backward(self._tok(x, mb), e.executor_resident_grads(x)))
            if self.K > 1:
                torch.mean(self.loss_parts, dim=0, keepdim=True, out=self.loss_dev)  # loss report only
            return e.step(want_norm=want_norm)

    def forward_only(self, batch: int | None = None) -> None:
        """FP-only pass (streaming inference / KD teacher) over self.tok_dev:
        loss -> self.loss_dev; no backward, no update (NEXT-4)."""
        e = self.engine
        B = batch or self.batch
        mb = B // self.K
        for fa in self.flashes:
            if fa is not None:
                fa.set_batch(mb)
        gp = self.gpts
        loss = [self.loss_dev.data_ptr()] if self.K == 1 else \
            [self.loss_parts.data_ptr() + 4 * x for x in range(self.K)]
        with torch.cuda.stream(self.stream):
            for i in range(self.mc.n_layers):
                P = e.forward_pre(i)

                def fwd(x, i=i, P=P):
                    if i == 0:
                        gp[x].embed_forward(self._tok(x, mb), mb, e.resident()[0])
                    self._layer_fwd(x, i, P)
                self._run(i, fwd)
                e.forward_post(i)
            rp = e.resident()[0]
            self._run(self.mc.n_layers, lambda x: gp[x].head_forward(self._tok(x, mb), rp, loss[x]))
            if self.K > 1:
                torch.mean(self.loss_parts, dim=0, keepdim=True, out=self.loss_dev)
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
        for g in self.gpts:
            g.close()


def bf16_bits_to_f32(u16: np.ndarray) -> np.ndarray:
    return (u16.astype(np.uint32) << 16).view(np.float32)
