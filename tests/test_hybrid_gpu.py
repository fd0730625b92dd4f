"""R28 hybrid update (include/sh.h sh_config.hybrid_layers; R28): the lowest host-optimised
layers keep their states in host RAM but are updated on the GPU by K2S, the split-master AdamW.

Bars: K2S equals the CPU pool's split AdamW BITWISE (special values included); a training run with any
number of hybrid layers, any window and a ring smaller than the GPU set is bitwise the all-resident run
(params, m, v, compute copies, losses) -- the property PAPER.md:87 asks of every placement; the engine
really took the hybrid path (K2S launches, staging / write-back bytes as counted).
"""
import numpy as np
import pytest
import torch

from tests._common import TINY, engine_run, engine_state, states_bitwise_equal
from tests.test_kernels_gpu import _special

pytestmark = pytest.mark.gpu

sh = pytest.importorskip("paper_conf_sc_sunwqyhxw22_b200.sh")

STEPS = 3


@pytest.mark.parametrize("n,n_decay", [(1 << 20, 1 << 19), (65536 + 8, 4096), (8, 8), (3 * 4096 + 24, 0)])
def test_k2s_bitwise_equals_cpu_split_adam(n, n_decay):
    p, g, m, v = _special(n, seed=n + 7)
    hi = np.empty(n, np.uint16)
    lo = np.empty(n, np.uint16)
    sh.op_master_split_cpu(p, hi, lo, n)
    sc = sh.adam_scalars(1.5e-4, 0.9, 0.999, 1e-8, 0.01, 3)
    dev = torch.device("cuda")
    th = torch.from_numpy(hi.view(np.int16).copy()).to(dev)
    tl = torch.from_numpy(lo.view(np.int16).copy()).to(dev)
    tm, tv, tg = (torch.from_numpy(a.copy()).to(dev) for a in (m, v, g))
    for _ in range(2):  # twice: the second launch on the stream reuses the schedule counters
        sh.op_adamw_split_gpu(th, tl, tm, tv, tg, n, n_decay, sc)
        sh.op_adamw_split_cpu(hi, lo, m, v, g, n, n_decay, sc)
    torch.cuda.synchronize()
    assert np.array_equal(th.cpu().numpy().view(np.uint16), hi)
    assert np.array_equal(tl.cpu().numpy().view(np.uint16), lo)
    assert np.array_equal(tm.cpu().numpy().view(np.uint32), m.view(np.uint32))
    assert np.array_equal(tv.cpu().numpy().view(np.uint32), v.view(np.uint32))


@pytest.fixture(scope="module")
def resident():
    ref, losses, _ = engine_run(TINY, STEPS, TINY["L"], sh.SH_BF16_MIXED)
    st = engine_state(ref)
    ref.close()
    return st, losses


@pytest.mark.parametrize("window,hybrid,ring,flags", [
    (0, 1, 0, 0), (0, 4, 0, sh.SH_FLAG_POISON), (1, 2, 0, sh.SH_FLAG_POISON), (2, 1, 0, 0),
    (2, 2, 2, sh.SH_FLAG_POISON), (1, 3, 2, sh.SH_FLAG_DELAY_INJECT), (3, 5, 0, 0)])
def test_hybrid_bitwise_equals_resident(resident, window, hybrid, ring, flags):
    ref_state, ref_losses = resident
    L = TINY["L"]
    tr, losses, _ = engine_run(TINY, STEPS, window, sh.SH_BF16_MIXED, flags=flags, ring_slots=ring,
                               hybrid_layers=hybrid)
    try:
        ok, what = states_bitwise_equal(engine_state(tr), ref_state)
        assert ok, f"window {window} hybrid {hybrid} ring {ring}: {what} differs from resident"
        assert [np.float32(x).tobytes() for x in losses] == [np.float32(x).tobytes() for x in ref_losses]
        s = tr.engine.stats()
        k = min(hybrid, L - window)
        assert s["hybrid_layers"] == hybrid
        assert s["hybrid_updates"] == STEPS * k
        n_pad = sum((x + 127) // 128 * 128 for x in tr.mc.layer_numels())  # homogeneous layers
        assert s["hybrid_h2d_bytes"] == STEPS * k * 10 * n_pad
        assert s["hybrid_d2h_bytes"] == STEPS * k * 12 * n_pad
        if k == L - window:  # every host layer on the GPU: the CPU pool has nothing to do
            assert s["cpu_adam_elems"] == 0
    finally:
        tr.close()


def test_hybrid_window_change_mid_run_bitwise(resident):
    ref_state, _ = resident
    tr, _, _ = engine_run(TINY, STEPS, 1, sh.SH_BF16_MIXED, hybrid_layers=1, set_window_at={1: 2, 2: 0})
    try:
        ok, what = states_bitwise_equal(engine_state(tr), ref_state)
        assert ok, what
    finally:
        tr.close()


@pytest.mark.parametrize("kw", [dict(precision=sh.SH_FP32), dict(max_grad_norm=0.5),
                                dict(flags=sh.SH_FLAG_FETCH_FP32)])
def test_hybrid_rejects_unsupported_modes(kw):
    prec = kw.pop("precision", sh.SH_BF16_MIXED)
    with pytest.raises(sh.ShError) as e:
        tr, _, _ = engine_run(TINY, 1, 1, prec, hybrid_layers=1, **kw)
        tr.close()
    assert e.value.status == sh.SH_ERR_INVALID
