"""Pins for the CPU oracle (oracle/gpt_oracle.py) against things other than itself.

No GPU.  Each pin is chosen so that a plausible slip in the oracle (dropped term,
wrong sign or index, transposed operand) fails at least one of them:
  * central finite differences, every parameter of a micro model (catches any
    backward error independent of the forward's correctness);
  * a model assembled from torch.nn.functional library routines in float64 and
    differentiated by autograd (catches forward definition errors: mask side,
    scale, LN variance bias, tied head, GELU variant, loss normalisation);
  * special cases with closed forms (seq=1 attention, zero final LN => ln V,
    constant-row LN == beta);
  * AdamW closed form under a constant gradient and torch.optim.AdamW float64.
"""
import math

import numpy as np
import pytest
import torch

import synth
from oracle import gpt_oracle as O


def micro(seed=7, L=2, h=16, nh=2, s=8, V=32):
    cfg = O.GPTConfig(L=L, h=h, nh=nh, s=s, V=V)
    layers = [[a.astype(np.float64) for a in synth.init_layer(seed, i, L, h)] for i in range(L)]
    # perturb biases / LN params so that every gradient path is exercised
    rng = np.random.default_rng(seed)
    for P in layers:
        for k in (0, 1, 3, 5, 6, 7, 9, 11):
            P[k] = P[k] + 0.1 * rng.standard_normal(P[k].shape)
        for k in (2, 4, 8, 10):
            P[k] = P[k] * 5.0  # larger weights => non-trivial attention / GELU regime
    res = [a.astype(np.float64) for a in synth.init_resident(seed, V, s, h)]
    res[0] = res[0] * 10
    res[2] = res[2] + 0.1 * rng.standard_normal(h)
    res[3] = res[3] + 0.1 * rng.standard_normal(h)
    tok = synth.tokens(0, 2, s, V, base_seed=seed)
    return cfg, layers, res, tok


def test_finite_difference_every_parameter():
    cfg, layers, res, tok = micro()
    loss0, gl, gr = O.forward_backward(cfg, layers, res, tok)
    eps = 1e-6
    worst = 0.0
    for tensors, grads in [(P, g) for P, g in zip(layers, gl)] + [(res, gr)]:
        for T, G in zip(tensors, grads):
            flat = T.reshape(-1)
            fd = np.empty_like(flat)
            for j in range(flat.size):
                old = flat[j]
                flat[j] = old + eps
                lp = _loss(cfg, layers, res, tok)
                flat[j] = old - eps
                lm = _loss(cfg, layers, res, tok)
                flat[j] = old
                fd[j] = (lp - lm) / (2 * eps)
            err = np.abs(fd - G.reshape(-1)).max() / max(np.abs(fd).max(), 1e-12)
            worst = max(worst, err)
            assert err < 1e-6, (T.shape, err)
    assert worst < 1e-6


def _loss(cfg, layers, res, tok):
    """Forward only (loss), reusing the oracle's forward ops."""
    wte, wpe, g, b = res
    inp, tgt = tok[:, :-1], tok[:, 1:]
    x = wte[inp] + wpe[np.arange(inp.shape[1])][None]
    for P in layers:
        x, _ = O.block_fwd(x, P, cfg.nh)
    xf, _ = O.layernorm_fwd(x, g, b)
    lg = xf @ wte.T
    z = lg - lg.max(-1, keepdims=True)
    logp = z - np.log(np.exp(z).sum(-1, keepdims=True))
    return -np.take_along_axis(logp, tgt[..., None], -1).mean()


def _torch_model_loss(cfg, layers, res, tok):
    """The same GPT built from torch.nn.functional library routines (float64)."""
    F = torch.nn.functional
    tl = [[torch.tensor(a, dtype=torch.float64, requires_grad=True) for a in P] for P in layers]
    tr = [torch.tensor(a, dtype=torch.float64, requires_grad=True) for a in res]
    t = torch.tensor(tok, dtype=torch.long)
    inp, tgt = t[:, :-1], t[:, 1:]
    B, S = inp.shape
    h, nh = cfg.h, cfg.nh
    x = F.embedding(inp, tr[0]) + tr[1][:S][None]
    for P in tl:
        a = F.layer_norm(x, (h,), P[0], P[1], eps=1e-5)
        qkv = F.linear(a, P[2], P[3])
        q, k, v = qkv.split(h, dim=-1)
        q, k, v = [z.view(B, S, nh, h // nh).transpose(1, 2) for z in (q, k, v)]
        o = F.scaled_dot_product_attention(q, k, v, is_causal=True)
        o = o.transpose(1, 2).reshape(B, S, h)
        x = x + F.linear(o, P[4], P[5])
        m = F.layer_norm(x, (h,), P[6], P[7], eps=1e-5)
        x = x + F.linear(F.gelu(F.linear(m, P[8], P[9]), approximate="tanh"), P[10], P[11])
    xf = F.layer_norm(x, (h,), tr[2], tr[3], eps=1e-5)
    logits = xf @ tr[0].T
    loss = F.cross_entropy(logits.reshape(B * S, -1), tgt.reshape(-1))
    loss.backward()
    return loss.item(), [[p.grad.numpy() for p in P] for P in tl], [p.grad.numpy() for p in tr]


@pytest.mark.parametrize("shape", [dict(L=2, h=16, nh=2, s=8, V=32), dict(L=1, h=32, nh=4, s=16, V=50)])
def test_forward_backward_vs_torch_functional(shape):
    cfg, layers, res, tok = micro(seed=11, **shape)
    loss, gl, gr = O.forward_backward(cfg, layers, res, tok)
    tloss, tgl, tgr = _torch_model_loss(cfg, layers, res, tok)
    assert abs(loss - tloss) < 1e-12 * max(1.0, abs(tloss))
    for a, b in zip([g for P in gl for g in P] + gr, [g for P in tgl for g in P] + tgr):
        assert np.abs(a - b).max() <= 1e-10 * max(np.abs(b).max(), 1e-30)


def test_attention_seq1_is_value_projection():
    rng = np.random.default_rng(0)
    qkv = rng.standard_normal((3, 1, 3 * 8))
    out, _ = O.attention_fwd(qkv, nh=2)
    assert np.array_equal(out, qkv[..., 16:])


def test_causal_first_token_attends_only_itself():
    rng = np.random.default_rng(1)
    qkv = rng.standard_normal((2, 5, 3 * 8))
    out, (_, _, _, p, _) = O.attention_fwd(qkv, nh=2)
    assert np.allclose(out[:, 0], qkv[:, 0, 16:], rtol=0, atol=1e-15)
    assert np.all(p[..., 0, 1:] == 0.0)  # -inf mask => exact zeros above the diagonal
    assert np.allclose(p.sum(-1), 1.0, atol=1e-14)


def test_zero_final_ln_gives_log_vocab_and_uniform_dlogits():
    cfg, layers, res, tok = micro(seed=3)
    res = [r.copy() for r in res]
    res[2][:] = 0.0
    res[3][:] = 0.0  # LN_f output == 0 -> logits == 0 -> uniform softmax
    loss, gl, gr = O.forward_backward(cfg, layers, res, tok)
    assert abs(loss - math.log(cfg.V)) < 1e-14
    # d loss / d lnf_b = sum_t dlogits_t @ E / N with dlogits = (1/V - onehot)/N
    N = tok.shape[0] * (tok.shape[1] - 1)
    tgt = tok[:, 1:].reshape(-1)
    dl = np.full((N, cfg.V), 1.0 / cfg.V)
    dl[np.arange(N), tgt] -= 1.0
    expect = (dl / N @ res[0]).sum(0)
    assert np.allclose(gr[3], expect, rtol=0, atol=1e-14)


def test_layernorm_constant_row_is_beta():
    x = np.full((4, 16), 3.25)
    g = np.linspace(0.5, 2.0, 16)
    b = np.linspace(-1, 1, 16)
    y, _ = O.layernorm_fwd(x, g, b)
    assert np.allclose(y, b, atol=0, rtol=0)


def test_gelu_known_values():
    # GELU_tanh(0) = 0; large positive -> identity; large negative -> 0; odd part: g(u) - g(-u) = u
    u = np.array([0.0, 10.0, -10.0, 1.0, -1.0])
    y = O.gelu_fwd(u)
    assert y[0] == 0.0 and abs(y[1] - 10.0) < 1e-12 and abs(y[2]) < 1e-12
    assert abs((y[3] - y[4]) - 1.0) < 1e-15
    assert abs(y[3] - 0.8411919906082768) < 1e-15  # 0.5(1+tanh(sqrt(2/pi)*1.044715))


def test_adamw_closed_form_constant_gradient():
    opt = O.AdamWConfig(lr=1e-2, weight_decay=0.0)
    g = np.array([0.3, -2.0, 1e-3])
    p = np.array([1.0, -0.5, 0.25])
    m = np.zeros(3); v = np.zeros(3)
    p0 = p.copy()
    for t in range(1, 11):
        p, m, v = O.adamw_update(p, g, m, v, t, opt, decay=False)
        # constant g => m_hat = g, v_hat = g^2 exactly => step = lr*g/(|g|+eps)
        expect = p0 - t * opt.lr * g / (np.abs(g) + opt.eps)
        assert np.allclose(p, expect, rtol=0, atol=1e-13)
    opt = O.AdamWConfig(lr=1e-2, weight_decay=0.1)
    p = p0.copy(); m = np.zeros(3); v = np.zeros(3)
    a = 1 - opt.lr * opt.weight_decay
    c = opt.lr * g / (np.abs(g) + opt.eps)
    for t in range(1, 11):
        p, m, v = O.adamw_update(p, g, m, v, t, opt, decay=True)
        expect = a ** t * p0 - c * (1 - a ** t) / (1 - a)
        assert np.allclose(p, expect, rtol=0, atol=1e-13)


def test_adamw_vs_torch_optim():
    rng = np.random.default_rng(5)
    p = rng.standard_normal(257)
    opt = O.AdamWConfig(lr=3e-3, weight_decay=0.05)
    tp = torch.tensor(p.copy(), requires_grad=True)
    topt = torch.optim.AdamW([tp], lr=opt.lr, betas=(opt.beta1, opt.beta2), eps=opt.eps,
                             weight_decay=opt.weight_decay)
    m = np.zeros_like(p); v = np.zeros_like(p)
    for t in range(1, 6):
        g = rng.standard_normal(257) * 10 ** rng.uniform(-6, 0)
        tp.grad = torch.tensor(g)
        topt.step()
        p, m, v = O.adamw_update(p, g, m, v, t, opt, decay=True)
        assert np.allclose(p, tp.detach().numpy(), rtol=0, atol=1e-15)


def test_grad_norm_and_clip_coef():
    gl = [[np.array([3.0, 0.0]), np.array([[4.0]])]]
    assert O.global_grad_norm(gl) == 5.0
    opt = O.AdamWConfig(lr=1.0, weight_decay=0.0, max_grad_norm=1.0)
    # clipped gradient enters Adam scaled by coef; with m=v=0 step-1 update = lr*g/(|g|+eps)
    p, m, v = O.adamw_update(np.array([0.0]), np.array([2.0]), np.zeros(1), np.zeros(1), 1, opt, False, coef=0.5)
    assert abs(m[0] - 0.1) < 1e-15 and abs(p[0] + 1.0 / (1.0 + 1e-8)) < 1e-15
