"""Shared test helpers: the tiny configuration (BASELINE.json configs[0]) and runners.

Parity metric (reading R16): after k steps, for every offload unit (a layer, or the
resident set) the ∞-norm relative error max|x - y| / max|y| over all its parameters, with y
the fp64 oracle.  Per-tensor values are reported as diagnostics.
"""
from __future__ import annotations

import numpy as np

import synth
from oracle import gpt_oracle as O

TINY = dict(L=4, h=256, nh=4, s=128, b=2, V=512)
FP32_TOL = 1e-4   # BASELINE.json north_star (fp32)
BF16_TOL = 2e-2   # BASELINE.json north_star (bf16 mixed)


def oracle_run(cfg: dict, steps: int, seed=1234, max_grad_norm=0.0, lr=1.5e-4, tok_seed=1234):
    c = O.GPTConfig(cfg["L"], cfg["h"], cfg["nh"], cfg["s"], cfg["V"])
    layers = [synth.init_layer(seed, i, cfg["L"], cfg["h"]) for i in range(cfg["L"])]
    res = synth.init_resident(seed, cfg["V"], cfg["s"], cfg["h"])
    st = O.make_state(layers, res)
    opt = O.AdamWConfig(lr=lr, max_grad_norm=max_grad_norm)
    losses, norms = [], []
    for t in range(steps):
        tok = synth.tokens(t, cfg["b"], cfg["s"], cfg["V"], base_seed=tok_seed)
        loss, norm, _ = O.train_step(c, st, tok, opt, synth.layer_weight_decay(cfg["h"]),
                                     synth.resident_weight_decay())
        losses.append(loss)
        norms.append(norm)
    return st, losses, norms


def unit_errors(eng_layers, eng_res, st):
    """Per offload unit ∞-norm relative error and per-tensor diagnostics."""
    out = {}
    for i, (E, Y) in enumerate(zip(eng_layers, st.layers)):
        num = max(float(np.abs(e.astype(np.float64) - y).max()) for e, y in zip(E, Y))
        den = max(float(np.abs(y).max()) for y in Y)
        out[f"layer{i}"] = num / den
    num = max(float(np.abs(e.astype(np.float64) - y).max()) for e, y in zip(eng_res, st.resident))
    den = max(float(np.abs(y).max()) for y in st.resident)
    out["resident"] = num / den
    return out


def engine_run(cfg: dict, steps: int, window: int, precision: int, seed=1234, max_grad_norm=0.0, lr=1.5e-4,
               flags=0, tok_seed=1234, set_window_at=None, cpu_threads=0, grad_ring_depth=0, attention="auto",
               ring_slots=0, executors=1, **kw):
    """Run the CUDA path; returns (trainer, losses, norms) with the trainer still open."""
    from paper_conf_sc_sunwqyhxw22_b200 import trainer as T
    mc = T.ModelConfig(cfg["L"], cfg["h"], cfg["nh"], cfg["s"], cfg["V"])
    tr = T.StrongholdTrainer(mc, batch=cfg["b"], window=window, precision=precision, lr=lr,
                             max_grad_norm=max_grad_norm, seed=seed, flags=flags, cpu_threads=cpu_threads,
                             grad_ring_depth=grad_ring_depth, attention=attention, ring_slots=ring_slots,
                             executors=executors, **kw)
    losses, norms = [], []
    for t in range(steps):
        if set_window_at and t in set_window_at:
            v = set_window_at[t]
            tr.engine.set_window(*v) if isinstance(v, tuple) else tr.engine.set_window(v)
        tr.set_tokens(synth.tokens(t, cfg["b"], cfg["s"], cfg["V"], base_seed=tok_seed))
        norms.append(tr.step_device(want_norm=True))
        losses.append(tr.loss())
    return tr, losses, norms


def engine_state(tr):
    """All layers + resident: (params, m, v) as lists of tensor lists (fp32)."""
    from paper_conf_sc_sunwqyhxw22_b200 import sh
    L = tr.mc.n_layers
    out = {}
    for what, name in ((sh.SH_READ_PARAM, "p"), (sh.SH_READ_M, "m"), (sh.SH_READ_V, "v")):
        out[name] = [tr.read_layer_tensors(i, what) for i in range(L)] + [tr.read_layer_tensors(-1, what)]
    out["c"] = [tr.engine.read_layer(i, sh.SH_READ_COMPUTE) for i in range(L)] + \
               [tr.engine.read_layer(-1, sh.SH_READ_COMPUTE)]
    return out


def states_bitwise_equal(a, b):
    for key in ("p", "m", "v"):
        for ua, ub in zip(a[key], b[key]):
            for x, y in zip(ua, ub):
                if x.view(np.uint32).tobytes() != y.view(np.uint32).tobytes():
                    return False, key
    for x, y in zip(a["c"], b["c"]):
        if x.tobytes() != y.tobytes():
            return False, "compute"
    return True, ""
