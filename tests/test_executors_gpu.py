"""NEXT-3 multi-stream executors (Fig. 5) on the GPU.

K training workers share ONE copy of every layer's parameters (the engine's ring slot), each
runs a micro-batch of batch/K sequences on its own CUDA stream, and the engine's K4 kernel
averages their gradients ("an all-reduce operation to synchronize the gradients among parallel
training workers before performing parameter updates") before the update.

Bars: (i) the same parity bar as the single-worker path against the fp64 oracle on the full
batch (data-parallel training within one GPU is the same math: "does not affect the model
consistency since parameter update takes after the entire batch has been processed",
PAPER.md:236); (ii) windowed == all-resident BITWISE with K workers (K4's fixed order keeps the
bit-exact-across-window invariant); (iii) concurrent workers give the same bits on every run.
"""
import pytest

from tests._common import (BF16_TOL, FP32_TOL, TINY, engine_run, engine_state, oracle_run, states_bitwise_equal,
                           unit_errors)

pytestmark = pytest.mark.gpu

sh = pytest.importorskip("paper_conf_sc_sunwqyhxw22_b200.sh")

STEPS = 3
TINY_B4 = dict(TINY, b=4)


def _errors(tr, st):
    L = tr.mc.n_layers
    return unit_errors([tr.read_layer_tensors(i) for i in range(L)], tr.read_layer_tensors(-1), st)


@pytest.fixture(scope="module")
def oracle_b4():
    return oracle_run(TINY_B4, STEPS)


@pytest.mark.parametrize("executors,window", [(2, 2), (4, 1), (4, TINY["L"])])
def test_executors_fp32_vs_oracle(oracle_b4, executors, window):
    st, olosses, onorms = oracle_b4
    tr, losses, norms = engine_run(TINY_B4, STEPS, window, sh.SH_FP32, executors=executors)
    try:
        errs = _errors(tr, st)
        assert max(errs.values()) <= FP32_TOL, errs
        for a, b in zip(losses, olosses):
            assert abs(a - b) <= 1e-5 * abs(b), (losses, olosses)
        for a, b in zip(norms, onorms):
            assert abs(a - b) <= 1e-4 * b, (norms, onorms)
    finally:
        tr.close()


def test_executors_bf16_flash_vs_oracle(oracle_b4):
    st, olosses, _ = oracle_b4
    tr, losses, _ = engine_run(TINY_B4, STEPS, 2, sh.SH_BF16_MIXED, executors=2, attention="flash")
    try:
        assert all(f is not None for f in tr.flashes)
        errs = _errors(tr, st)
        assert max(errs.values()) <= BF16_TOL, errs
        for a, b in zip(losses, olosses):
            assert abs(a - b) <= 2e-2 * abs(b)
    finally:
        tr.close()


@pytest.mark.parametrize("precision", [sh.SH_FP32, sh.SH_BF16_MIXED])
def test_executors_windowed_bitwise_equals_resident(precision):
    L = TINY["L"]
    ref_tr, ref_losses, ref_norms = engine_run(TINY_B4, STEPS, L, precision, executors=2)
    ref = engine_state(ref_tr)
    ref_tr.close()
    for w in range(0, L):
        tr, losses, norms = engine_run(TINY_B4, STEPS, w, precision, executors=2)
        try:
            ok, what = states_bitwise_equal(engine_state(tr), ref)
            assert ok, f"window {w}: {what} differs from the all-resident run"
            assert losses == ref_losses and norms == ref_norms
        finally:
            tr.close()


def test_executors_repeatable_and_close_to_single_worker():
    a, la, _ = engine_run(TINY_B4, 2, 1, sh.SH_FP32, executors=4)
    sa = engine_state(a)
    a.close()
    b, lb, _ = engine_run(TINY_B4, 2, 1, sh.SH_FP32, executors=4)
    sb = engine_state(b)
    b.close()
    ok, what = states_bitwise_equal(sa, sb)
    assert ok and la == lb, what  # concurrent streams, same bits
    c, lc, _ = engine_run(TINY_B4, 2, 1, sh.SH_FP32, executors=1)
    c.close()
    for x, y in zip(la, lc):  # same math, different summation split
        assert abs(x - y) <= 1e-5 * abs(y)


def test_executor_grads_protocol():
    from paper_conf_sc_sunwqyhxw22_b200 import trainer as T
    mc = T.ModelConfig(TINY["L"], TINY["h"], TINY["nh"], TINY["s"], TINY["V"])
    tr = T.StrongholdTrainer(mc, batch=4, window=2, precision=sh.SH_FP32, executors=2)
    try:
        with pytest.raises(sh.ShError):
            tr.engine.executor_grads(0, 1)  # not between a backward PRE and POST
        with pytest.raises(sh.ShError):
            tr.engine.executor_grads(0, 2)  # executor out of range
        with pytest.raises(ValueError):
            T.StrongholdTrainer(mc, batch=3, window=2, precision=sh.SH_FP32, executors=2)
    finally:
        tr.close()


def test_executors_clip_fp32_vs_oracle():
    """Clip mode: the global norm is taken over the executors' AVERAGED gradients (K4 runs before K3)."""
    st, _, onorms = oracle_run(TINY_B4, STEPS, max_grad_norm=0.5)
    assert onorms[0] > 0.5
    tr, _, norms = engine_run(TINY_B4, STEPS, 1, sh.SH_FP32, max_grad_norm=0.5, executors=2)
    try:
        errs = _errors(tr, st)
        assert max(errs.values()) <= FP32_TOL, errs
        for a, b in zip(norms, onorms):
            assert abs(a - b) <= 1e-4 * b, (norms, onorms)
    finally:
        tr.close()
