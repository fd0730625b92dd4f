"""CPU-only checks of the native boundary: the C-ABI libraries load, export every function the
headers declare, and the host-side pieces (CPU AdamW of the pool, bf16 RNE shadow writer,
layout/argument validation, Adam scalars) are correct without a GPU."""
import ctypes
import math
import os
import re
import subprocess

import numpy as np
import pytest
import torch

import synth
from tests._common import rna_bf16_bits
from oracle import gpt_oracle as O

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sh = pytest.importorskip("paper_conf_sc_sunwqyhxw22_b200.sh")
gpt = pytest.importorskip("paper_conf_sc_sunwqyhxw22_b200.gpt")


def _declared(header):
    text = open(os.path.join(ROOT, "include", header)).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return set(re.findall(r"\b((?:sh|gpt)_[a-z0-9_]+)\s*\(", text))


@pytest.mark.parametrize("header,libname,py", [("sh.h", "libsh.so", "sh"), ("sh_gpt.h", "libsh_gpt.so", "gpt")])
def test_library_exports_every_declared_symbol(header, libname, py):
    decl = _declared(header)
    assert decl, header
    path = os.path.join(ROOT, "paper_conf_sc_sunwqyhxw22_b200", "lib", libname)
    out = subprocess.run(["nm", "-D", "--defined-only", path], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\sT\s(\w+)", out))
    missing = decl - exported
    assert not missing, missing
    lib = ctypes.CDLL(path)
    for name in decl:
        getattr(lib, name)
    mod = sh if py == "sh" else gpt
    assert decl == set(mod.EXPORTS), decl ^ set(mod.EXPORTS)


def test_abi_version_and_error_string():
    assert sh.lib().sh_abi_version() == 3
    with pytest.raises(sh.ShError) as e:
        sh.adam_scalars(1e-3, 0.9, 0.999, 1e-8, 0.0, 0)  # t must be >= 1
    assert e.value.status == sh.SH_ERR_INVALID and "t must be" in str(e.value)


def test_adam_scalars_rounded_once_from_double():
    s = sh.adam_scalars(1.5e-4, 0.9, 0.999, 1e-8, 0.01, 3)
    assert s.step_size == np.float32(1.5e-4 / (1 - 0.9 ** 3))
    assert s.sqrt_bc2 == np.float32(math.sqrt(1 - 0.999 ** 3))
    assert s.decay == np.float32(1 - 1.5e-4 * 0.01)
    assert s.omb1 == np.float32(1 - 0.9) and s.omb2 == np.float32(1 - 0.999)
    assert s.beta1 == np.float32(0.9) and s.eps == np.float32(1e-8)


@pytest.mark.parametrize("n,n_decay", [(1 << 16, 1 << 15), (8, 0), (4096 + 8, 4096 + 8), (100008, 40000)])
def test_cpu_adam_matches_oracle_and_is_thread_invariant(n, n_decay):
    p, g, m, v = synth.random_adam_state(n, n)
    sc = sh.adam_scalars(1e-3, 0.9, 0.999, 1e-8, 0.05, 4)
    outs = []
    for threads in (1, 3, 8):
        cp, cm, cv = p.copy(), m.copy(), v.copy()
        c16 = np.empty(n, np.uint16)
        sh.op_adamw_cpu(cp, cm, cv, g, c16, n, n_decay, sc, threads=threads)
        outs.append((cp, cm, cv, c16))
    for o in outs[1:]:
        for a, b in zip(o, outs[0]):
            assert a.tobytes() == b.tobytes()  # bitwise identical for any thread split
    cp, cm, cv, c16 = outs[0]
    opt = O.AdamWConfig(lr=1e-3, weight_decay=0.05)
    dec = np.arange(n) < n_decay
    for d in (True, False):
        if not (dec == d).any():
            continue
        rp, rm, rv = O.adamw_update(p[dec == d].astype(np.float64), g[dec == d].astype(np.float64),
                                    m[dec == d].astype(np.float64), v[dec == d].astype(np.float64), 4, opt, d)
        # fp32 rounding of each op (and of the fp32 scalars) relative to the element's scale
        scale = np.abs(p[dec == d]) + np.abs(rp - p[dec == d])
        assert (np.abs(cp[dec == d] - rp) <= 1e-6 * scale + 1e-30).all()
        assert np.abs(cm[dec == d] - rm).max() <= 1e-6 * np.abs(rm).max()
        assert np.abs(cv[dec == d] - rv).max() <= 1e-6 * np.abs(rv).max()
    # the shadow is the bf16 (RNA, R25) of the new master
    assert np.array_equal(c16, rna_bf16_bits(cp))


def test_cpu_adam_clip_coefficient_scales_gradient():
    n = 4096
    p, g, m, v = synth.random_adam_state(3, n)
    sc = sh.adam_scalars(1e-3, 0.9, 0.999, 1e-8, 0.0, 1)
    a = [x.copy() for x in (p, m, v)]
    b = [x.copy() for x in (p, m, v)]
    sh.op_adamw_cpu(a[0], a[1], a[2], g, None, n, 0, sc, coef=0.25)
    g4 = (g * np.float32(0.25)).astype(np.float32)
    sh.op_adamw_cpu(b[0], b[1], b[2], g4, None, n, 0, sc)
    for x, y in zip(a, b):
        assert x.tobytes() == y.tobytes()


def _special_values():
    x = synth.normal(synth.stream_key(1, 2), 1 << 15, 10.0)
    x[:10] = [np.nan, -np.nan, np.inf, -np.inf, 0.0, -0.0, 1e-40, -1e-41, 3.3895314e38, 1.0000001]
    ties = ((np.arange(1, 200, dtype=np.uint32) << 16) | 0x8000).view(np.float32)  # exact ties, both parities
    x[10:10 + ties.size] = ties
    x[300:300 + ties.size] = -ties
    return x, ties


def test_bf16_rna_cpu_matches_reference_and_canonical_nan():
    x, ties = _special_values()
    d = np.empty(x.size, np.uint16)
    sh.op_cast_bf16_cpu(x, d, x.size)
    assert d[0] == 0x7FC0 and d[1] == 0x7FC0
    assert np.array_equal(d, rna_bf16_bits(x))
    # round to nearest: equal to torch's RNE everywhere except exact ties with an even truncation, where
    # RNA moves away from zero; no result is farther than half a bf16 ulp from x
    rne = torch.from_numpy(x[2:]).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
    diff = d[2:] != rne
    u = x[2:].view(np.uint32)
    assert np.array_equal(diff, ((u & 0xFFFF) == 0x8000) & ((u >> 16) & 1 == 0))
    fin = np.isfinite(x[2:]) & np.isfinite((d[2:].astype(np.uint32) << 16).view(np.float32))
    r = (d[2:].astype(np.uint32) << 16).view(np.float32)[fin].astype(np.float64)
    ulp = np.abs(np.spacing(r.astype(np.float32)).astype(np.float64)) * 2 ** 16
    assert (np.abs(r - x[2:][fin]) <= 0.5 * ulp + 1e-45).all()


def test_split_master_is_lossless():
    """R25: hi = the compute copy (RNA), lo = the low 16 bits; join(split(p)) == p for every non-NaN fp32
    pattern (specials, ties of both parities, random bit patterns), NaN -> NaN."""
    x, _ = _special_values()
    rnd = synth.uniform_u64(synth.stream_key(9, 9), 1 << 16).astype(np.uint32).view(np.float32)
    x = np.concatenate([x, rnd, (np.arange(0, 1 << 16, dtype=np.uint32) | 0x3F800000).view(np.float32)])
    n = x.size
    hi, lo, back = np.empty(n, np.uint16), np.empty(n, np.uint16), np.empty(n, np.float32)
    sh.op_master_split_cpu(x, hi, lo, n)
    sh.op_master_join_cpu(hi, lo, back, n)
    assert np.array_equal(hi, rna_bf16_bits(x))
    assert np.array_equal(lo, (x.view(np.uint32) & 0xFFFF).astype(np.uint16))
    ok = ~np.isnan(x)
    assert np.array_equal(back[ok].view(np.uint32), x[ok].view(np.uint32))
    assert np.isnan(back[~ok]).all()


@pytest.mark.parametrize("coef", [None, 0.3])
def test_cpu_adam_on_split_master_equals_fp32(coef):
    """The pool's AdamW on a split master == the fp32 AdamW bitwise (joined p, m, v) and hi == its bf16."""
    n, n_decay = 1 << 16, 1 << 15
    p, g, m, v = synth.random_adam_state(11, n)
    sc = sh.adam_scalars(1e-3, 0.9, 0.999, 1e-8, 0.01, 5)
    a = [x.copy() for x in (p, m, v)]
    s16 = np.empty(n, np.uint16)
    sh.op_adamw_cpu(a[0], a[1], a[2], g, s16, n, n_decay, sc, coef=coef, threads=3)
    hi, lo = np.empty(n, np.uint16), np.empty(n, np.uint16)
    sh.op_master_split_cpu(p, hi, lo, n)
    bm, bv = m.copy(), v.copy()
    sh.op_adamw_split_cpu(hi, lo, bm, bv, g, n, n_decay, sc, coef=coef, threads=2)
    back = np.empty(n, np.float32)
    sh.op_master_join_cpu(hi, lo, back, n)
    assert back.tobytes() == a[0].tobytes() and bm.tobytes() == a[1].tobytes() and bv.tobytes() == a[2].tobytes()
    assert np.array_equal(hi, s16)


def test_op_argument_validation():
    a = np.zeros(16, np.float32)
    sc = sh.adam_scalars(1e-3, 0.9, 0.999, 1e-8, 0.0, 1)
    with pytest.raises(sh.ShError) as e:
        sh.op_adamw_cpu(a, a.copy(), a.copy(), a.copy(), None, 12, 0, sc)  # n not a multiple of 8
    assert e.value.status == sh.SH_ERR_INVALID


def test_engine_init_rejects_bad_config_without_touching_gpu():
    with pytest.raises(sh.ShError) as e:
        sh.Engine([[8, 8]], [[1, 0]], [8], [1], window=5, stream=1)  # window > n_layers
    assert e.value.status == sh.SH_ERR_INVALID
    with pytest.raises(sh.ShError) as e:
        sh.Engine([[8, 0]], [[1, 0]], [8], [1], window=0, stream=1)  # zero-size tensor
    assert e.value.status == sh.SH_ERR_INVALID
    with pytest.raises(sh.ShError) as e:
        sh.Engine([[8]], [[1]], [8], [1], window=0, stream=None)  # compute stream required
    assert e.value.status == sh.SH_ERR_INVALID
    with pytest.raises(sh.ShError) as e:
        sh.Engine([[8]], [[1]], [8], [1], window=0, stream=1, max_grad_norm=1.0, grad_ring_depth=1,
                  )  # clip mode needs a landing buffer per layer: ok with L=1 ... then fails on CUDA
    assert e.value.status in (sh.SH_ERR_CUDA, sh.SH_ERR_INVALID, sh.SH_ERR_OOM_HOST)
