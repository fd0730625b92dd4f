"""Ragged and degenerate shapes on the CUDA path (padding of every tensor to 128 elements, head dim
24, odd batch, a single-layer model).  Same bars as test_engine_gpu: fp32 / bf16 against the fp64
oracle per offload unit after 3 steps, windowed == resident bitwise for every window."""
import numpy as np
import pytest

from tests._common import (BF16_TOL, FP32_TOL, engine_run, engine_state, oracle_run, states_bitwise_equal,
                           unit_errors)

pytestmark = pytest.mark.gpu
sh = pytest.importorskip("paper_conf_sc_sunwqyhxw22_b200.sh")

RAGGED = dict(L=3, h=72, nh=3, s=24, b=3, V=104)   # no tensor is a multiple of 128 elements
SINGLE = dict(L=1, h=64, nh=2, s=16, b=1, V=64)    # one layer: window 0 or 1 only
STEPS = 3


def _errs(tr, st, cfg):
    return unit_errors([tr.read_layer_tensors(i) for i in range(cfg["L"])], tr.read_layer_tensors(-1), st)


@pytest.mark.parametrize("cfg", [RAGGED, SINGLE], ids=["ragged", "single_layer"])
def test_vs_oracle_and_bitwise_windows(cfg):
    st, olosses, _ = oracle_run(cfg, STEPS)
    L = cfg["L"]
    for precision, tol in ((sh.SH_FP32, FP32_TOL), (sh.SH_BF16_MIXED, BF16_TOL)):
        ref, losses, _ = engine_run(cfg, STEPS, L, precision)
        try:
            errs = _errs(ref, st, cfg)
            assert max(errs.values()) <= tol, (precision, errs)
            if precision == sh.SH_FP32:
                for a, b in zip(losses, olosses):
                    assert abs(a - b) <= 1e-5 * abs(b)
            ref_state = engine_state(ref)
        finally:
            ref.close()
        for w in range(L):
            for flags in (0, sh.SH_FLAG_FETCH_FP32 if precision == sh.SH_BF16_MIXED else sh.SH_FLAG_POISON):
                tr, _, _ = engine_run(cfg, STEPS, w, precision, flags=flags)
                try:
                    ok, what = states_bitwise_equal(engine_state(tr), ref_state)
                    assert ok, (precision, w, flags, what)
                finally:
                    tr.close()


def test_ragged_clip_mode_matches_oracle():
    st, _, onorms = oracle_run(RAGGED, STEPS, max_grad_norm=0.25)
    assert onorms[0] > 0.25
    tr, _, norms = engine_run(RAGGED, STEPS, 1, sh.SH_FP32, max_grad_norm=0.25)
    try:
        assert max(_errs(tr, st, RAGGED).values()) <= FP32_TOL
        for a, b in zip(norms, onorms):
            assert abs(a - b) <= 1e-4 * b
    finally:
        tr.close()


def test_clip_inactive_equals_no_clip_bitwise():
    """max_grad_norm above the gradient norm: coef == 1 exactly, so clip mode must reproduce the
    no-clip run bit for bit (g * 1.0f == g)."""
    a, _, _ = engine_run(RAGGED, STEPS, 1, sh.SH_BF16_MIXED, max_grad_norm=1e9)
    b, _, _ = engine_run(RAGGED, STEPS, 1, sh.SH_BF16_MIXED)
    try:
        ok, what = states_bitwise_equal(engine_state(a), engine_state(b))
        assert ok, what
    finally:
        a.close()
        b.close()
