"""CPU oracle: one plain fp64 GPT training step with AdamW, no offloading.

TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs may import this module.  It shares no code
with the CUDA path (paper_conf_sc_sunwqyhxw22_b200/) and imports nothing from it.

What it computes and why this is the right oracle
-------------------------------------------------
STRONGHOLD's claim is that offloading "do[es] not introduce stale model updates
nor ... affect the training precision" (§III-A).  So the windowed
engine must reach exactly what ordinary synchronous training reaches: this file
is that definition written out -- a GPT-like model (§V-B,
"GPT-like Transformer-based models [35],[3]"; reading R1 in DESIGN.md: GPT-2
pre-LN, tied embedding, learned positions, tanh-GELU), mean token cross entropy,
hand-derived backward, Adam [22] with decoupled weight decay (
reading R2), optional global-norm clipping (reading R3).  All arithmetic is
float64; numpy.matmul / exp / tanh are the only library primitives.  Layer-wise
activation checkpointing changes no value, so it is not modelled.

Pins (tests/test_oracle.py, all `-m "not gpu"`):
  * gradients: central finite differences on a micro model, every parameter;
  * forward + gradients vs a model assembled from torch.nn.functional library
    routines in float64 with autograd;
  * special cases: seq=1 attention == V projection; zero head => loss == ln V;
    constant-row LayerNorm == beta;
  * AdamW: closed form for a constant gradient; torch.optim.AdamW in float64.

Layouts: x is [B, S, h]; weights follow y = x @ W.T + b (W is [out, in]);
qkv columns are [q | k | v], head j owns columns j*hd:(j+1)*hd of each.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

LN_EPS = 1e-5  # GPT-2 LayerNorm epsilon (reading R1)


@dataclass
class GPTConfig:
    L: int
    h: int
    nh: int
    s: int
    V: int


@dataclass
class AdamWConfig:
    """Reading R2: Megatron GPT-2 / ZeRO-Offload defaults (PAPER.md:265 cites [23],[11])."""
    lr: float = 1.5e-4
    beta1: float = 0.9
    beta2: float = 0.999
    eps: float = 1e-8
    weight_decay: float = 0.01
    max_grad_norm: float = 0.0  # <= 0: no clipping (reading R3)


# ----------------------------------------------------------------------------- ops

def layernorm_fwd(x, g, b):
    """LN(z) = (z - mu)/sqrt(var + eps) * g + b, biased variance (reading R1)."""
    mu = x.mean(axis=-1, keepdims=True)
    var = ((x - mu) ** 2).mean(axis=-1, keepdims=True)
    rstd = 1.0 / np.sqrt(var + LN_EPS)
    xhat = (x - mu) * rstd
    return xhat * g + b, (xhat, rstd)


def layernorm_bwd(dy, cache, g):
    xhat, rstd = cache
    red = tuple(range(dy.ndim - 1))
    dg = (dy * xhat).sum(axis=red)
    db = dy.sum(axis=red)
    dxhat = dy * g
    dx = rstd * (dxhat - dxhat.mean(axis=-1, keepdims=True)
                 - xhat * (dxhat * xhat).mean(axis=-1, keepdims=True))
    return dx, dg, db


_GELU_C = math.sqrt(2.0 / math.pi)


def gelu_fwd(u):
    """GELU_tanh(u) = 0.5 u (1 + tanh(sqrt(2/pi)(u + 0.044715 u^3)))."""
    return 0.5 * u * (1.0 + np.tanh(_GELU_C * (u + 0.044715 * u ** 3)))


def gelu_bwd(du, u):
    t = np.tanh(_GELU_C * (u + 0.044715 * u ** 3))
    dt = (1.0 - t * t) * _GELU_C * (1.0 + 3.0 * 0.044715 * u * u)
    return du * (0.5 * (1.0 + t) + 0.5 * u * dt)


def attention_fwd(qkv, nh):
    """Causal multi-head self attention: S = Q K^T / sqrt(hd), P = softmax(S) with
    -inf above the diagonal (max-subtracted), O = P V.  qkv: [B, S, 3h]."""
    B, S, h3 = qkv.shape
    h = h3 // 3
    hd = h // nh
    q = qkv[..., 0:h].reshape(B, S, nh, hd).transpose(0, 2, 1, 3)
    k = qkv[..., h:2 * h].reshape(B, S, nh, hd).transpose(0, 2, 1, 3)
    v = qkv[..., 2 * h:].reshape(B, S, nh, hd).transpose(0, 2, 1, 3)
    scale = 1.0 / math.sqrt(hd)
    sc = (q @ k.transpose(0, 1, 3, 2)) * scale
    mask = np.triu(np.ones((S, S), dtype=bool), k=1)
    sc = np.where(mask, -np.inf, sc)
    sc = sc - sc.max(axis=-1, keepdims=True)
    e = np.exp(sc)
    p = e / e.sum(axis=-1, keepdims=True)
    o = p @ v  # [B, nh, S, hd]
    out = o.transpose(0, 2, 1, 3).reshape(B, S, h)
    return out, (q, k, v, p, scale)


def attention_bwd(dout, cache):
    q, k, v, p, scale = cache
    B, nh, S, hd = q.shape
    do = dout.reshape(B, S, nh, hd).transpose(0, 2, 1, 3)
    dv = p.transpose(0, 1, 3, 2) @ do
    dp = do @ v.transpose(0, 1, 3, 2)
    ds = p * (dp - (dp * p).sum(axis=-1, keepdims=True))  # softmax Jacobian
    dq = (ds @ k) * scale
    dk = (ds.transpose(0, 1, 3, 2) @ q) * scale
    def merge(t):
        return t.transpose(0, 2, 1, 3).reshape(B, S, nh * hd)
    return np.concatenate([merge(dq), merge(dk), merge(dv)], axis=-1)


def linear_fwd(x, W, b):
    return x @ W.T + b


def linear_bwd(dy, x, W):
    d2 = dy.reshape(-1, dy.shape[-1])
    x2 = x.reshape(-1, x.shape[-1])
    return dy @ W, d2.T @ x2, d2.sum(axis=0)


# ------------------------------------------------------------------------- model

def block_fwd(x, P, nh):
    """One pre-LN GPT-2 block.  P = [ln1_g, ln1_b, w_qkv, b_qkv, w_o, b_o,
    ln2_g, ln2_b, w_fc, b_fc, w_proj, b_proj] (SURVEY §8(a) a0 packed order)."""
    a, c_ln1 = layernorm_fwd(x, P[0], P[1])
    qkv = linear_fwd(a, P[2], P[3])
    o, c_att = attention_fwd(qkv, nh)
    x1 = x + linear_fwd(o, P[4], P[5])
    m, c_ln2 = layernorm_fwd(x1, P[6], P[7])
    f = linear_fwd(m, P[8], P[9])
    g = gelu_fwd(f)
    x2 = x1 + linear_fwd(g, P[10], P[11])
    return x2, (a, c_ln1, qkv, o, c_att, m, c_ln2, f, g)


def block_bwd(dx2, cache, P):
    a, c_ln1, qkv, o, c_att, m, c_ln2, f, g = cache
    dg, dWproj, dbproj = linear_bwd(dx2, g, P[10])
    df = gelu_bwd(dg, f)
    dm, dWfc, dbfc = linear_bwd(df, m, P[8])
    dx1_ln, dg2, db2 = layernorm_bwd(dm, c_ln2, P[6])
    dx1 = dx2 + dx1_ln
    do, dWo, dbo = linear_bwd(dx1, o, P[4])
    dqkv = attention_bwd(do, c_att)
    da, dWqkv, dbqkv = linear_bwd(dqkv, a, P[2])
    dx_ln, dg1, db1 = layernorm_bwd(da, c_ln1, P[0])
    dx = dx1 + dx_ln
    return dx, [dg1, db1, dWqkv, dbqkv, dWo, dbo, dg2, db2, dWfc, dbfc, dWproj, dbproj]


def forward_backward(cfg: GPTConfig, layers, resident, tok):
    """Loss and gradients of one batch.  tok: int [B, S+1]; inputs tok[:, :S],
    targets tok[:, 1:]; loss = mean over all B*S tokens of -log softmax(logits)[target]
    (reading R1; PAPER.md:49 describes FP -> loss -> BP -> update)."""
    wte, wpe, lnf_g, lnf_b = resident
    inp, tgt = tok[:, :-1], tok[:, 1:]
    B, S = inp.shape
    x = wte[inp] + wpe[np.arange(S)][None, :, :]
    caches = []
    for P in layers:
        x, c = block_fwd(x, P, cfg.nh)
        caches.append(c)
    xf, c_lnf = layernorm_fwd(x, lnf_g, lnf_b)
    logits = xf @ wte.T  # tied head
    z = logits - logits.max(axis=-1, keepdims=True)
    lse = np.log(np.exp(z).sum(axis=-1, keepdims=True))
    logp = z - lse
    N = B * S
    loss = -np.take_along_axis(logp, tgt[..., None], axis=-1).sum() / N
    # backward
    dlogits = np.exp(logp)
    np.put_along_axis(dlogits, tgt[..., None], np.take_along_axis(dlogits, tgt[..., None], -1) - 1.0, -1)
    dlogits /= N
    dxf = dlogits @ wte
    dwte = dlogits.reshape(N, -1).T @ xf.reshape(N, -1)
    dx, dlnf_g, dlnf_b = layernorm_bwd(dxf, c_lnf, lnf_g)
    grads = [None] * len(layers)
    for i in range(len(layers) - 1, -1, -1):
        dx, grads[i] = block_bwd(dx, caches[i], layers[i])
    np.add.at(dwte, inp.reshape(-1), dx.reshape(N, -1))  # lookup + tied-head contributions
    dwpe = np.zeros_like(wpe)
    dwpe[:S] = dx.sum(axis=0)
    return loss, grads, [dwte, dwpe, dlnf_g, dlnf_b]


# --------------------------------------------------------------------- optimizer

def global_grad_norm(grad_lists):
    """||g||_2 over every parameter (reading R3), float64."""
    return math.sqrt(sum(float((g.astype(np.float64) ** 2).sum()) for gl in grad_lists for g in gl))


def adamw_update(p, g, m, v, t, opt: AdamWConfig, decay: bool, coef: float = 1.0):
    """Adam (Kingma & Ba [22], Alg. 1) with decoupled weight decay, step t >= 1:
       g <- coef*g;  m <- b1 m + (1-b1) g;  v <- b2 v + (1-b2) g^2;
       p <- p (1 - lr*lambda) - (lr/bc1) m / (sqrt(v)/sqrt(bc2) + eps),  bc_k = 1 - b_k^t.
    Returns new (p, m, v) in float64."""
    g = g * coef
    m = opt.beta1 * m + (1.0 - opt.beta1) * g
    v = opt.beta2 * v + (1.0 - opt.beta2) * g * g
    bc1 = 1.0 - opt.beta1 ** t
    bc2 = 1.0 - opt.beta2 ** t
    if decay:
        p = p * (1.0 - opt.lr * opt.weight_decay)
    p = p - (opt.lr / bc1) * m / (np.sqrt(v) / math.sqrt(bc2) + opt.eps)
    return p, m, v


@dataclass
class OracleState:
    layers: list
    resident: list
    m_layers: list = field(default_factory=list)
    v_layers: list = field(default_factory=list)
    m_res: list = field(default_factory=list)
    v_res: list = field(default_factory=list)
    t: int = 0


def make_state(layers_f32, resident_f32) -> OracleState:
    L = [[np.asarray(a, dtype=np.float64).copy() for a in P] for P in layers_f32]
    R = [np.asarray(a, dtype=np.float64).copy() for a in resident_f32]
    return OracleState(L, R,
                       [[np.zeros_like(a) for a in P] for P in L], [[np.zeros_like(a) for a in P] for P in L],
                       [np.zeros_like(a) for a in R], [np.zeros_like(a) for a in R])


def train_step(cfg: GPTConfig, st: OracleState, tok, opt: AdamWConfig, layer_wd, res_wd):
    """One synchronous training iteration: FP, loss, BP, (clip), AdamW on every
    parameter.  Mutates st; returns (loss, grad_norm, grads)."""
    loss, gl, gr = forward_backward(cfg, st.layers, st.resident, tok)
    norm = global_grad_norm(gl + [gr])
    coef = 1.0
    if opt.max_grad_norm > 0:
        coef = min(1.0, opt.max_grad_norm / (norm + 1e-6))
    st.t += 1
    for i, P in enumerate(st.layers):
        for k in range(len(P)):
            P[k], st.m_layers[i][k], st.v_layers[i][k] = adamw_update(
                P[k], gl[i][k], st.m_layers[i][k], st.v_layers[i][k], st.t, opt, layer_wd[k], coef)
    for k in range(len(st.resident)):
        st.resident[k], st.m_res[k], st.v_res[k] = adamw_update(
            st.resident[k], gr[k], st.m_res[k], st.v_res[k], st.t, opt, res_wd[k], coef)
    return loss, norm, (gl, gr)
