"""Heterogeneous offload units through the C-ABI alone (no GPT driver): layers of very different
sizes and tensor counts (the offload unit is whatever the user calls a layer;
P:195: models "with a heterogeneous layer structure").  Every ring slot is sized for the largest
unit, so small units must come and go through the same slots as large ones.

The "model" is a toy whose backward writes g = c * a_t + b_k (two IEEE fp32 ops on the compute
copy c the engine hands out: fp32 master, or its bf16 (RNA) copy), so the host side can reproduce
every gradient exactly with plain PyTorch CPU ops and the fp64 oracle AdamW
(oracle.gpt_oracle.adamw_update) gives the reference parameters.  Bars: engine vs oracle per unit
(∞-norm relative ≤ 1e-5 after 3 steps), and every window / decoupled ring bitwise equal to the
all-resident run."""
import numpy as np
import pytest
import torch

from oracle import gpt_oracle as O
from tests._common import rna_bf16_f32

pytestmark = pytest.mark.gpu
sh = pytest.importorskip("paper_conf_sc_sunwqyhxw22_b200.sh")

LAYERS = [[1000, 24], [70000, 64, 1], [200], [5000, 100, 8, 3000], [64], [30000, 3000], [7]]
WD = [[1, 0], [1, 0, 0], [1], [1, 1, 0, 0], [0], [1, 0], [1]]
RES, RES_WD = [512, 16], [1, 0]
STEPS = 3
LR = 1e-3


class _Dev:
    """A device buffer the engine owns, seen by torch through __cuda_array_interface__."""

    def __init__(self, ptr, n, typestr):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (int(ptr), False),
                                         "version": 2, "strides": None}


def _view(ptr, n, bf16):
    if bf16:
        return torch.as_tensor(_Dev(ptr, n, "<i2"), device="cuda").view(torch.bfloat16)
    return torch.as_tensor(_Dev(ptr, n, "<f4"), device="cuda")


def _coef(t, layer, k):
    a = np.float32(0.5 + 0.1 * t)
    b = np.float32(1e-3 * (1 + layer) * (-1) ** k)
    return a, b


def _init():
    rng = np.random.default_rng(7)
    return ([[rng.standard_normal(n).astype(np.float32) * np.float32(0.02) for n in lay] for lay in LAYERS],
            [rng.standard_normal(n).astype(np.float32) * np.float32(0.02) for n in RES])


def _engine_run(window, precision, ring_slots=0, ring_bytes=0, stats=None, flags=0):
    bf16 = precision == sh.SH_BF16_MIXED
    stream = torch.cuda.Stream()
    eng = sh.Engine(LAYERS, WD, RES, RES_WD, window=window, precision=precision, lr=LR, stream=stream,
                    ring_slots=ring_slots, cpu_threads=4, ring_bytes=ring_bytes, flags=flags)
    try:
        lay, res = _init()
        for i, ts in enumerate(lay):
            eng.register(i, np.concatenate(ts))
        eng.register(-1, np.concatenate(res))
        L = len(LAYERS)
        for t in range(STEPS):
            with torch.cuda.stream(stream):
                for i in range(L):
                    eng.forward_pre(i)
                    eng.forward_post(i)
                for i in reversed(range(L)):
                    P, G = eng.backward_pre(i)
                    for k, n in enumerate(LAYERS[i]):
                        a, b = _coef(t, i, k)
                        c = _view(P[k], n, bf16).float()
                        _view(G[k], n, False).add_(c * float(a) + float(b))
                    eng.backward_post(i)
                rp, rg = eng.resident()
                for k, n in enumerate(RES):
                    a, b = _coef(t, L, k)
                    c = _view(rp[k], n, bf16).float()
                    _view(rg[k], n, False).add_(c * float(a) + float(b))
            eng.step()
        eng.synchronize()
        if stats is not None:
            stats.update(eng.stats())
        out = [eng.read_layer(i, w) for i in range(L) for w in (sh.SH_READ_PARAM, sh.SH_READ_M, sh.SH_READ_V)]
        out += [eng.read_layer(-1, w) for w in (sh.SH_READ_PARAM, sh.SH_READ_M, sh.SH_READ_V)]
        return out
    finally:
        eng.close()


def _oracle(bf16):
    """fp64 AdamW on the exactly reproduced gradients; params as fp64 arrays per unit (caller order)."""
    lay, res = _init()
    units = [list(u) for u in lay] + [list(res)]
    wds = WD + [RES_WD]
    opt = O.AdamWConfig(lr=LR)
    p = [[x.astype(np.float64) for x in u] for u in units]
    m = [[np.zeros_like(x) for x in u] for u in p]
    v = [[np.zeros_like(x) for x in u] for u in p]
    for t in range(STEPS):
        for i, u in enumerate(p):
            for k, x in enumerate(u):
                a, b = _coef(t, i, k)
                c = torch.from_numpy(x.astype(np.float32))
                if bf16:  # the engine's compute copy: bf16 round-to-nearest, ties away (R25)
                    c = torch.from_numpy(rna_bf16_f32(x.astype(np.float32)))
                g = (c * float(a) + float(b)).numpy().astype(np.float64)
                p[i][k], m[i][k], v[i][k] = O.adamw_update(x, g, m[i][k], v[i][k], t + 1, opt, bool(wds[i][k]))
    return [np.concatenate(u) for u in p]


@pytest.mark.parametrize("precision", ["SH_FP32", "SH_BF16_MIXED"])
def test_heterogeneous_units_vs_oracle_and_bitwise_windows(precision):
    prec = getattr(sh, precision)
    L = len(LAYERS)
    ref = _engine_run(L, prec)
    want = _oracle(prec == sh.SH_BF16_MIXED)
    for i, w in enumerate(want):
        got = ref[3 * i]
        err = np.abs(got - w).max() / np.abs(w).max()
        assert err <= 1e-5, (i, err)
    runs = [(w, 0) for w in range(L)] + [(5, 3), (L, 2)]  # + decoupled rings smaller than the window
    for w, ring in runs:
        out = _engine_run(w, prec, ring)
        for k, (x, y) in enumerate(zip(out, ref)):
            assert x.tobytes() == y.tobytes(), (w, ring, k // 3, k % 3)


def _pad(n):
    return (n + 127) // 128 * 128


@pytest.mark.parametrize("precision", ["SH_FP32", "SH_BF16_MIXED"])
def test_fixed_byte_window_heterogeneous(precision):
    """NEXT-4 fixed-byte window: one buffer of ring_bytes holds a variable number of
    layers.  2.5 largest-layer slots of bytes hold 5 slots here (the largest, then layers 1-4 at
    their own sizes), where fixed-size slots would hold 2; training is bitwise the resident run's
    for any GPU-optimised set, with slot poisoning on (a slot reused by a smaller layer must never
    expose stale bytes)."""
    prec = getattr(sh, precision)
    L = len(LAYERS)
    cb = 2 if prec == sh.SH_BF16_MIXED else 4
    npad = [sum(_pad(n) for n in lay) for lay in LAYERS]
    slot = lambda n: (cb * n + 255) // 256 * 256 + (4 * n + 255) // 256 * 256  # noqa: E731
    budget = int(2.5 * slot(max(npad)))
    caps, total = [max(npad)], slot(max(npad))
    for x in range(1, L):
        if total + slot(npad[x]) > budget:
            break
        caps.append(npad[x])
        total += slot(npad[x])
    assert len(caps) >= 4  # many more layers than the 2 fixed-size slots the same bytes would hold
    ref = _engine_run(L, prec)
    for w in (0, 1, 3, 6):
        st = {}
        out = _engine_run(w, prec, ring_bytes=budget, stats=st, flags=sh.SH_FLAG_POISON)
        assert st["n_slots"] == len(caps) and st["ring_bytes"] == total <= budget, (st["n_slots"], st["ring_bytes"])
        for k, (x, y) in enumerate(zip(out, ref)):
            assert x.tobytes() == y.tobytes(), (w, k // 3, k % 3)


def test_fixed_byte_window_rejects_too_small_and_autotune():
    stream = torch.cuda.Stream()
    with pytest.raises(sh.ShError) as e:
        sh.Engine(LAYERS, WD, RES, RES_WD, window=0, precision=sh.SH_FP32, stream=stream, ring_bytes=4096)
    assert e.value.status == sh.SH_ERR_INVALID and "largest layer" in str(e.value)
    with pytest.raises(sh.ShError) as e:
        sh.Engine(LAYERS, WD, RES, RES_WD, window=-1, precision=sh.SH_FP32, stream=stream, ring_bytes=1 << 30)
    assert e.value.status == sh.SH_ERR_INVALID
