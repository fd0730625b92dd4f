"""The parity bars can fail (VERDICT r01 "make parity able to fail"), CPU only.

The engine-vs-oracle tests (tests/test_engine_gpu.py, test_parity_l8_gpu.py, test_dp_host_gpu.py)
use the per-tensor update-delta bar of tests/_common.py (R24).  Here, without a GPU:
  * an honest float32 run of the same algorithm (the oracle's steps on float32 arrays -- the
    precision of the CUDA path's fp32 mode) PASSES the fp32 bars, so they are not tighter than
    fp32 arithmetic allows;
  * plausible optimizer bugs FAIL them: every update skipped, the step-2 bias-correction scalars
    reused at step 3, one update applied twice, the gradient sign flipped on one tensor;
  * the round-1 per-unit bar (max|x - y| / max|y|, dominated by LN gamma = 1) lets the first two
    through -- the reason the delta bar exists.
"""
import math

import numpy as np
import pytest

import synth
from oracle import gpt_oracle as O
from tests._common import (BF16_TOL, DELTA_BF16, DELTA_FP32, FP32_TOL, KBIAS_MAX, TINY, delta_errors, grad_errors,
                           init_state, kbias_bound, oracle_run, unit_errors)

STEPS = 3
LR = 1.5e-4


def _run(dtype, steps=STEPS, t_override=None, twice_at=None, flip=None):
    """The oracle's training loop on `dtype` arrays with optional mutations:
    t_override {step: t} -- bias-correction step used by the update at `step` (1-based);
    twice_at -- the update of that step is applied twice;  flip -- (layer, tensor) whose gradient
    sign is flipped."""
    cfg = TINY
    c = O.GPTConfig(cfg["L"], cfg["h"], cfg["nh"], cfg["s"], cfg["V"])
    L0, R0 = init_state(cfg)
    Ls = [[np.array(a, dtype) for a in U] for U in L0]
    Rs = [np.array(a, dtype) for a in R0]
    mL = [[np.zeros_like(a) for a in U] for U in Ls]
    vL = [[np.zeros_like(a) for a in U] for U in Ls]
    mR = [np.zeros_like(a) for a in Rs]
    vR = [np.zeros_like(a) for a in Rs]
    opt = O.AdamWConfig(lr=LR)
    lwd, rwd = synth.layer_weight_decay(cfg["h"]), synth.resident_weight_decay()
    g1 = None
    for step in range(1, steps + 1):
        tok = synth.tokens(step - 1, cfg["b"], cfg["s"], cfg["V"])
        _, gl, gr = O.forward_backward(c, Ls, Rs, tok)
        if step == 1:
            g1 = (gl, gr)
        if flip is not None:
            gl[flip[0]][flip[1]] = -gl[flip[0]][flip[1]]
        t = (t_override or {}).get(step, step)
        for _ in range(2 if twice_at == step else 1):
            for i, U in enumerate(Ls):
                for k in range(len(U)):
                    U[k], mL[i][k], vL[i][k] = O.adamw_update(U[k], gl[i][k], mL[i][k], vL[i][k], t, opt, lwd[k])
                    U[k], mL[i][k], vL[i][k] = U[k].astype(dtype), mL[i][k].astype(dtype), vL[i][k].astype(dtype)
            for k in range(len(Rs)):
                Rs[k], mR[k], vR[k] = O.adamw_update(Rs[k], gr[k], mR[k], vR[k], t, opt, rwd[k])
                Rs[k], mR[k], vR[k] = Rs[k].astype(dtype), mR[k].astype(dtype), vR[k].astype(dtype)
    return Ls, Rs, g1


@pytest.fixture(scope="module")
def ref():
    st, _, _, g1 = oracle_run(TINY, STEPS, lr=LR, keep_grads=True)
    return st, g1


def _worst(d):
    return max(d.values())


def test_fp32_arithmetic_passes_the_fp32_bars(ref):
    st, g1 = ref
    x0 = init_state(TINY)
    Ls, Rs, g1x = _run(np.float32)
    d = delta_errors(Ls, Rs, x0, st.layers, st.resident)
    assert _worst(d) <= DELTA_FP32, sorted(d.items(), key=lambda kv: -kv[1])[:5]
    assert kbias_bound(Ls, x0[0], STEPS, LR) <= KBIAS_MAX
    assert _worst(unit_errors(Ls, Rs, st)) <= FP32_TOL
    ge, kb = grad_errors(g1x[0], g1x[1], g1[0], g1[1])
    assert _worst(ge) <= 1e-4, sorted(ge.items(), key=lambda kv: -kv[1])[:5]
    assert kb <= 1e-4  # the K-bias gradient is rounding noise next to the Q/V-bias gradients


def test_skipped_updates_fail_the_delta_bar_but_passed_the_unit_bar(ref):
    st, _ = ref
    x0 = init_state(TINY)
    d = delta_errors(x0[0], x0[1], x0, st.layers, st.resident)
    assert min(d.values()) >= 0.99  # nothing moved: 100 % error on every tensor
    assert _worst(d) > DELTA_BF16
    # the round-1 bf16 bar let a run without any update through
    assert _worst(unit_errors(x0[0], x0[1], st)) <= BF16_TOL


def test_stale_bias_correction_fails_the_fp32_delta_bar_but_passed_the_unit_bar(ref):
    st, _ = ref
    x0 = init_state(TINY)
    Ls, Rs, _ = _run(np.float64, t_override={3: 2})
    d = delta_errors(Ls, Rs, x0, st.layers, st.resident)
    assert _worst(d) > 10 * DELTA_FP32, _worst(d)
    assert _worst(unit_errors(Ls, Rs, st)) <= FP32_TOL  # invisible to the round-1 bar


def test_double_update_fails_both_delta_bars(ref):
    st, _ = ref
    x0 = init_state(TINY)
    Ls, Rs, _ = _run(np.float64, twice_at=2)
    d = delta_errors(Ls, Rs, x0, st.layers, st.resident)
    assert _worst(d) > DELTA_BF16


def test_flipped_gradient_sign_on_one_tensor_fails(ref):
    st, _ = ref
    x0 = init_state(TINY)
    Ls, Rs, _ = _run(np.float64, flip=(2, 8))  # layer 2's W_fc
    d = delta_errors(Ls, Rs, x0, st.layers, st.resident)
    assert d["layer2.W_fc"] > 1.0  # (later steps see a different model, so other tensors move too)
    # the per-unit bar only sees it through the unit max
    assert _worst(unit_errors(Ls, Rs, st)) > FP32_TOL


def test_kbias_bound_catches_garbage():
    x0 = init_state(TINY)
    Ls = [[a.copy() for a in U] for U in x0[0]]
    h = TINY["h"]
    Ls[1][3][h:2 * h] += 5 * LR  # a K bias moved by more than three Adam steps can
    assert kbias_bound(Ls, x0[0], STEPS, LR) > KBIAS_MAX
    assert math.isclose(kbias_bound(x0[0], x0[0], STEPS, LR), 0.0)
