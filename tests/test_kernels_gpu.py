"""K1 / K2 / K3 on the GPU through the C-ABI op entry points (sh_op_*).

K2 (GPU AdamW) must equal the CPU AdamW of the pool BITWISE -- the property that makes the
engine's results independent of which layers the GPU updates (every window size).
Both are also checked against the fp64 oracle AdamW (oracle/gpt_oracle.adamw_update).
"""
import numpy as np
import pytest
import torch

import synth
from oracle import gpt_oracle as O
from tests._common import rna_bf16_bits

pytestmark = pytest.mark.gpu

sh = pytest.importorskip("paper_conf_sc_sunwqyhxw22_b200.sh")


def _special(n, seed):
    p, g, m, v = synth.random_adam_state(seed, n)
    # special values: zeros, denormals, huge, exact bf16 ties, negative zero
    k = min(64, n // 8)
    g[:k] = 0.0
    g[k:2 * k] = np.float32(1e-40)  # denormal gradient
    p[2 * k:3 * k] = np.float32(1e-39)  # denormal parameter
    p[3 * k:4 * k] = np.float32(3.0e38)
    ties = (np.arange(k, dtype=np.uint32) << 16) | 0x8000  # exactly half-way between two bf16
    p[4 * k:5 * k] = (ties | 0x3F800000 & 0xFFFF0000).view(np.float32)
    p[5 * k:6 * k] = -0.0
    v[6 * k:7 * k] = 0.0
    return p, g, m, v


@pytest.mark.parametrize("n,n_decay,use_coef,out", [(1 << 20, 1 << 19, False, "bf16"), (65536 + 8, 4096, True, "bf16"),
                                                      (8, 8, False, "fp32"), (3 * 2048 + 16, 0, True, "fp32")])
def test_k2_bitwise_equals_cpu_adam(n, n_decay, use_coef, out):
    p, g, m, v = _special(n, seed=n)
    sc = sh.adam_scalars(1.5e-4, 0.9, 0.999, 1e-8, 0.01, 3)
    coef = np.float32(0.37)
    dev = torch.device("cuda")
    tp, tm, tv, tg = (torch.from_numpy(a.copy()).to(dev) for a in (p, m, v, g))
    t16 = torch.empty(n, dtype=torch.int16, device=dev)
    t32 = torch.empty(n, dtype=torch.float32, device=dev)
    tcoef = torch.tensor([coef], device=dev)
    sh.op_adamw_gpu(tp, tm, tv, tg, t16 if out == "bf16" else None, t32 if out == "fp32" else None, n, n_decay, sc,
                    coef=tcoef if use_coef else None)
    torch.cuda.synchronize()
    cp, cm, cv = p.copy(), m.copy(), v.copy()
    c16 = np.empty(n, dtype=np.uint16)
    sh.op_adamw_cpu(cp, cm, cv, g, c16 if out == "bf16" else None, n, n_decay, sc, coef=coef if use_coef else None)
    for a, b in ((tp, cp), (tm, cm), (tv, cv)):
        assert np.array_equal(a.cpu().numpy().view(np.uint32), b.view(np.uint32))
    if out == "bf16":
        assert np.array_equal(t16.cpu().numpy().view(np.uint16), c16)
    else:
        assert np.array_equal(t32.cpu().numpy().view(np.uint32), cp.view(np.uint32))
    # and both follow the fp64 oracle AdamW to fp32 rounding
    opt = O.AdamWConfig(lr=1.5e-4, weight_decay=0.01)
    sel = slice(8 * 64, None)  # skip the special-value block
    dec = np.arange(n) < n_decay
    for d in (True, False):
        mask = dec[sel] == d
        if not mask.any():
            continue
        rp, rm, rv = O.adamw_update(p[sel][mask].astype(np.float64), g[sel][mask].astype(np.float64),
                                    m[sel][mask].astype(np.float64), v[sel][mask].astype(np.float64), 3, opt, d,
                                    coef=float(coef) if use_coef else 1.0)
        assert np.abs(cp[sel][mask] - rp).max() <= 1e-6 * max(1.0, np.abs(rp).max())


def test_k1_cast_matches_cpu_and_rna_reference():
    n = 1 << 16
    x = synth.normal(synth.stream_key(9, 9), n, 3.0)
    x[:8] = [np.nan, np.inf, -np.inf, 1e-40, -1e-40, 0.0, -0.0, 3.4e38]
    ties = ((np.arange(1, 200, dtype=np.uint32) << 16) | 0x8000).view(np.float32)
    x[8:8 + ties.size] = ties  # exact ties of both parities
    dev = torch.device("cuda")
    d16 = torch.empty(n, dtype=torch.int16, device=dev)
    sh.op_cast_bf16_gpu(torch.from_numpy(x).to(dev), d16, n)
    torch.cuda.synchronize()
    c16 = np.empty(n, dtype=np.uint16)
    sh.op_cast_bf16_cpu(x, c16, n)
    g16 = d16.cpu().numpy().view(np.uint16)
    assert np.array_equal(g16, c16)
    assert g16[0] == 0x7FC0
    assert np.array_equal(g16, rna_bf16_bits(x))  # torch's RNE + the ties-away rule (R25)


@pytest.mark.parametrize("n", [8, 1 << 12, (1 << 22) + 8, 50304 * 256])
def test_k3_sumsq_deterministic_and_exact(n):
    g = synth.normal(synth.stream_key(n, 5), n, 1e-3)
    dev = torch.device("cuda")
    tg = torch.from_numpy(g).to(dev)
    out = torch.zeros(2, dtype=torch.float64, device=dev)
    sh.op_sumsq_gpu(tg, n, out[0:1])
    sh.op_sumsq_gpu(tg, n, out[1:2])
    torch.cuda.synchronize()
    a, b = out.cpu().numpy()
    assert a.tobytes() == b.tobytes()
    exact = float(np.sum(g.astype(np.float64) ** 2))
    assert abs(a - exact) <= 1e-12 * exact


@pytest.mark.parametrize("n,k", [(8, 2), (1 << 12, 3), ((1 << 22) + 8, 4), (201379840 // 64 * 8, 8)])
def test_k4_exec_reduce_matches_plain_sum(n, k):
    """K4 (NEXT-3 executor all-reduce): ((g0 + g1) + ...) * fp32(1/k), bitwise equal to
    the same IEEE fp32 op sequence written with plain torch elementwise ops, and within fp32 rounding
    of the exact fp64 mean."""
    dev = torch.device("cuda")
    gs = [torch.from_numpy(synth.normal(synth.stream_key(n + e, 11), n, 1e-3)).to(dev) for e in range(k)]
    inv = np.float32(1.0 / k)
    ref = gs[0].clone()
    for e in range(1, k):
        ref = ref + gs[e]
    ref = ref * torch.tensor(inv, device=dev)
    mean64 = sum(g.double() for g in gs) / k
    dst = gs[0].clone()
    sh.op_exec_reduce_gpu(dst, gs[1:], n, float(inv))
    torch.cuda.synchronize()
    assert torch.equal(dst.view(torch.int32), ref.view(torch.int32))
    err = (dst.double() - mean64).abs().max().item()
    assert err <= k * 2.0 ** -23 * mean64.abs().max().item() + 1e-30
