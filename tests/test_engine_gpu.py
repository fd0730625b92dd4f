"""End-to-end parity of the CUDA path (engine + GPT driver) on the tiny configuration.

Bars (BASELINE.json north_star; R16, R24; tests/_common.py):
  * windowed == all-resident (w = L) BITWISE for every window 0..L: params, m, v, compute copies
  * vs the fp64 oracle after 3 steps, per TENSOR update delta ||dx - dy|| / ||dy|| <= 1e-3 (fp32),
    <= 5e-2 (bf16 mixed); K bias bounded by the Adam step bound; per offload unit max|x-y|/max|y|
    <= 1e-4 / 2e-2; loss per step within 1e-5 relative (fp32)
  * step-1 gradients per tensor vs the oracle (tests/test_parity_l8_gpu.py)
"""
import numpy as np
import pytest

import synth
from tests._common import (BF16_TOL, DELTA_BF16, DELTA_BF16_1D, DELTA_FP32, FP32_TOL, TINY, check_vs_oracle,
                           delta_errors, engine_run, engine_state, init_state, log_metric, oracle_run,
                           states_bitwise_equal, worst)

pytestmark = pytest.mark.gpu

sh = pytest.importorskip("paper_conf_sc_sunwqyhxw22_b200.sh")

STEPS = 3


@pytest.fixture(scope="module")
def oracle_noclip():
    return oracle_run(TINY, STEPS)


@pytest.fixture(scope="module")
def oracle_clip():
    return oracle_run(TINY, STEPS, max_grad_norm=0.5)


@pytest.mark.parametrize("window", [TINY["L"], 2])
def test_fp32_vs_oracle(oracle_noclip, window):
    st, olosses, onorms = oracle_noclip
    tr, losses, norms = engine_run(TINY, STEPS, window, sh.SH_FP32)
    try:
        check_vs_oracle(tr, st, DELTA_FP32, FP32_TOL, f"tiny_fp32_w{window}")
        for a, b in zip(losses, olosses):
            assert abs(a - b) <= 1e-5 * abs(b), (losses, olosses)
        for a, b in zip(norms, onorms):
            assert abs(a - b) <= 1e-4 * b, (norms, onorms)
    finally:
        tr.close()


def test_bf16_vs_oracle_and_noise_floor(oracle_noclip):
    """bf16 mixed through both attention cores of the GPT driver: each within the bf16 bars of the
    oracle, and the two correct bf16 implementations' mutual per-tensor delta logged as the bf16
    noise floor the 1-D bar is set from (R24)."""
    st, olosses, _ = oracle_noclip
    got, trs = {}, {}
    try:
        for attention in ("flash", "cublas"):
            tr, losses, _ = engine_run(TINY, STEPS, 2, sh.SH_BF16_MIXED, attention=attention)
            trs[attention] = tr
            assert (tr.flash is not None) == (attention == "flash")
            for a, b in zip(losses, olosses):
                assert abs(a - b) <= 2e-2 * abs(b)
            got[attention] = ([tr.read_layer_tensors(i) for i in range(TINY["L"])], tr.read_layer_tensors(-1))
        x0 = init_state(TINY)
        mutual = delta_errors(got["flash"][0], got["flash"][1], x0, got["cublas"][0], got["cublas"][1])
        m2 = delta_errors(got["flash"][0], got["flash"][1], x0, got["cublas"][0], got["cublas"][1], ndim=2)
        m1 = {k: v for k, v in mutual.items() if k not in m2}
        log_metric("tiny_bf16_flash_vs_cublas", mutual_worst_2d=worst(m2), mutual_worst_1d=worst(m1),
                   top=sorted(mutual.items(), key=lambda kv: -kv[1])[:8])
        for attention, tr in trs.items():
            check_vs_oracle(tr, st, DELTA_BF16, BF16_TOL, f"tiny_bf16_{attention}", delta_tol_1d=DELTA_BF16_1D)
    finally:
        for tr in trs.values():
            tr.close()


def test_clip_fp32_vs_oracle(oracle_clip):
    st, olosses, onorms = oracle_clip
    assert onorms[0] > 0.5  # clipping is active in this run
    tr, losses, norms = engine_run(TINY, STEPS, 1, sh.SH_FP32, max_grad_norm=0.5)
    try:
        check_vs_oracle(tr, st, DELTA_FP32, FP32_TOL, "tiny_fp32_clip")
        for a, b in zip(norms, onorms):
            assert abs(a - b) <= 1e-4 * b, (norms, onorms)
    finally:
        tr.close()


@pytest.mark.parametrize("precision", [sh.SH_FP32, sh.SH_BF16_MIXED])
def test_windowed_bitwise_equals_resident(precision):
    L = TINY["L"]
    ref, ref_losses, _ = engine_run(TINY, STEPS, L, precision)
    ref_state = engine_state(ref)
    ref.close()
    for w in range(0, L):
        tr, losses, _ = engine_run(TINY, STEPS, w, precision)
        try:
            ok, what = states_bitwise_equal(engine_state(tr), ref_state)
            assert ok, f"window {w}: {what} differs from resident"
            assert [np.float32(x).tobytes() for x in losses] == [np.float32(x).tobytes() for x in ref_losses]
            s = tr.engine.stats()
            if w < L:
                assert s["h2d_bytes"] > 0 and s["d2h_bytes"] > 0
        finally:
            tr.close()


def test_clip_windowed_bitwise_and_poison():
    L = TINY["L"]
    ref, _, _ = engine_run(TINY, STEPS, L, sh.SH_BF16_MIXED, max_grad_norm=0.5)
    ref_state = engine_state(ref)
    ref.close()
    for w, flags in ((0, 0), (2, sh.SH_FLAG_POISON), (3, sh.SH_FLAG_SYNC_CPU)):
        tr, _, _ = engine_run(TINY, STEPS, w, sh.SH_BF16_MIXED, max_grad_norm=0.5, flags=flags)
        try:
            ok, what = states_bitwise_equal(engine_state(tr), ref_state)
            assert ok, f"clip window {w} flags {flags}: {what}"
        finally:
            tr.close()


def test_fetch_fp32_mode_bitwise_equals_resident():
    """SH_FLAG_FETCH_FP32: no host shadow, fp32 master over the link, K1 cast on the GPU."""
    L = TINY["L"]
    ref, _, _ = engine_run(TINY, STEPS, L, sh.SH_BF16_MIXED)
    ref_state = engine_state(ref)
    ref.close()
    for w in (0, 1, 3):
        tr, _, _ = engine_run(TINY, STEPS, w, sh.SH_BF16_MIXED, flags=sh.SH_FLAG_FETCH_FP32 | sh.SH_FLAG_POISON)
        try:
            ok, what = states_bitwise_equal(engine_state(tr), ref_state)
            assert ok, f"window {w}: {what}"
            s = tr.engine.stats()
            # 4 B/param over the link: FP fetches L-w layers
            assert s["h2d_bytes"] % 4 == 0 and s["h2d_bytes"] > 0
        finally:
            tr.close()


def test_host_layouts_bitwise_equal_and_fetch_bytes():
    """The three bf16 host layouts train bitwise alike (the resident run has no host layout at all):
    split master (default, R25; fetch = hi plane, 2 B/param), fp32 master + bf16 shadow
    (SH_FLAG_BF16_SHADOW; 2 B/param), fp32 master (SH_FLAG_FETCH_FP32; 4 B/param + K1 cast).  Every
    prefetch of the split layout moves exactly the bf16 compute copy."""
    L, w = TINY["L"], 1
    ref, _, _ = engine_run(TINY, STEPS, L, sh.SH_BF16_MIXED)
    ref_state = engine_state(ref)
    ref.close()
    h2d = {}
    for name, flags in (("split", 0), ("shadow", sh.SH_FLAG_BF16_SHADOW), ("fp32", sh.SH_FLAG_FETCH_FP32)):
        tr, _, _ = engine_run(TINY, STEPS, w, sh.SH_BF16_MIXED, flags=flags | sh.SH_FLAG_POISON)
        try:
            ok, what = states_bitwise_equal(engine_state(tr), ref_state)
            assert ok, f"{name}: {what}"
            h2d[name] = tr.engine.stats()["h2d_bytes"]
        finally:
            tr.close()
    assert h2d["split"] == h2d["shadow"] and h2d["fp32"] == 2 * h2d["split"], h2d


def test_window_change_mid_run_bitwise():
    L = TINY["L"]
    ref, _, _ = engine_run(TINY, 4, L, sh.SH_BF16_MIXED)
    ref_state = engine_state(ref)
    ref.close()
    tr, _, _ = engine_run(TINY, 4, 1, sh.SH_BF16_MIXED, set_window_at={1: 3, 2: 0, 3: 2})
    try:
        ok, what = states_bitwise_equal(engine_state(tr), ref_state)
        assert ok, what
    finally:
        tr.close()


def test_small_landing_ring_and_one_thread_bitwise():
    L = TINY["L"]
    ref, _, _ = engine_run(TINY, STEPS, L, sh.SH_FP32)
    ref_state = engine_state(ref)
    ref.close()
    tr, _, _ = engine_run(TINY, STEPS, 1, sh.SH_FP32, cpu_threads=1, grad_ring_depth=1)
    try:
        ok, what = states_bitwise_equal(engine_state(tr), ref_state)
        assert ok, what
    finally:
        tr.close()


def test_lr_zero_leaves_params_unchanged():
    tr, _, _ = engine_run(TINY, 2, 1, sh.SH_FP32, lr=0.0)
    try:
        for i in range(TINY["L"]):
            got = tr.read_layer_tensors(i)
            init = synth.init_layer(1234, i, TINY["L"], TINY["h"])
            for a, b in zip(got, init):
                assert np.array_equal(a.view(np.uint32), b.view(np.uint32))
    finally:
        tr.close()


def test_protocol_errors():
    tr, _, _ = engine_run(TINY, 1, 1, sh.SH_FP32)
    try:
        with pytest.raises(sh.ShError) as e:
            tr.engine.forward_pre(1)  # must start at layer 0
        assert e.value.status == sh.SH_ERR_STATE
        with pytest.raises(sh.ShError):
            tr.engine.step()
        with pytest.raises(sh.ShError) as e:
            tr.engine.set_window(99)
        assert e.value.status == sh.SH_ERR_INVALID
        # the context is still usable after protocol errors
        tr.set_tokens(synth.tokens(5, TINY["b"], TINY["s"], TINY["V"]))
        tr.step_device()
        assert np.isfinite(tr.loss())
    finally:
        tr.close()


@pytest.mark.parametrize("precision", [sh.SH_FP32, sh.SH_BF16_MIXED])
def test_forward_only_passes(precision):
    """NEXT-4 FP-only streaming (KD teacher inference): the loss of an FP-only
    pass equals the training step's loss at the same parameters bitwise, for every window; passes
    update nothing; a training step after FP-only passes is unaffected by them."""
    L = TINY["L"]
    tok0 = synth.tokens(0, TINY["b"], TINY["s"], TINY["V"])
    ref, ref_losses, _ = engine_run(TINY, 2, L, precision)
    ref_state = engine_state(ref)
    ref.close()
    for w in (0, 1, L):
        from paper_conf_sc_sunwqyhxw22_b200 import trainer as T
        mc = T.ModelConfig(L, TINY["h"], TINY["nh"], TINY["s"], TINY["V"])
        tr = T.StrongholdTrainer(mc, batch=TINY["b"], window=w, precision=precision)
        try:
            tr.set_tokens(tok0)
            losses = []
            for _ in range(3):
                tr.forward_only()
                losses.append(np.float32(tr.loss()).tobytes())
            assert len(set(losses)) == 1 and losses[0] == np.float32(ref_losses[0]).tobytes(), w
            assert tr.engine.stats()["step"] == 0
            for t in range(2):  # training continues exactly as if the passes never happened
                tr.set_tokens(synth.tokens(t, TINY["b"], TINY["s"], TINY["V"]))
                tr.step_device(want_norm=True)
            ok, what = states_bitwise_equal(engine_state(tr), ref_state)
            assert ok, (w, what)
        finally:
            tr.close()


def test_autotune_mid_run_bitwise_and_trace():
    """window = -1: w0 = min(2, L) for the warm-up steps, then sh_autotune_window applies the solver
    on the measured profile (P1/P2 + eq. 3 with SH_FLAG_CPU_HARD); results stay bitwise equal to the
    resident run, and the step trace / overlap stats of the profiled steps are consistent."""
    L = TINY["L"]
    ref, _, _ = engine_run(TINY, 4, L, sh.SH_BF16_MIXED)
    ref_state = engine_state(ref)
    ref.close()
    from paper_conf_sc_sunwqyhxw22_b200 import trainer as T
    mc = T.ModelConfig(L, TINY["h"], TINY["nh"], TINY["s"], TINY["V"])
    tr = T.StrongholdTrainer(mc, batch=TINY["b"], window=-1, precision=sh.SH_BF16_MIXED, warmup_steps=2,
                             flags=sh.SH_FLAG_CPU_HARD | sh.SH_FLAG_PROFILE)
    try:
        for t in range(4):
            tr.set_tokens(synth.tokens(t, TINY["b"], TINY["s"], TINY["V"]))
            tr.step_device(want_norm=True)
        ok, what = states_bitwise_equal(engine_state(tr), ref_state)
        assert ok, what
        st = tr.engine.stats()
        assert 0 <= st["window"] <= L and st["profiled_steps"] >= 3
        prof = tr.engine.profile()
        assert all(x > 0 for x in prof["t_fp"]) and all(x > 0 for x in prof["t_bp"])
        trace = tr.engine.trace()
        kinds = {e["kind"] for e in trace}
        assert {"fp", "bp", "k2_adamw"} <= kinds
        fp = sorted((e["layer"], e["start_ms"], e["end_ms"]) for e in trace if e["kind"] == "fp")
        assert [x[0] for x in fp] == list(range(L))
        assert all(a[2] <= b[1] + 1e-3 for a, b in zip(fp, fp[1:]))  # FP layers run in order
        assert all(e["end_ms"] >= e["start_ms"] >= 0 for e in trace if e["kind"] not in ("cpu_adam", "h2d_wait_cpu"))
        # host-clock intervals (aligned to the step start; an issuer wait can begin before the GPU reaches it)
        host = [e for e in trace if e["kind"] in ("cpu_adam", "h2d_wait_cpu")]
        assert all(e["end_ms"] >= e["start_ms"] for e in host)
        if st["window"] < L:
            assert {e["layer"] for e in host if e["kind"] == "cpu_adam"} == set(range(st["window"], L))
        if st["window"] < L:
            assert 0.0 <= st["h2d_overlap_frac"] <= 1.0 and 0.0 <= st["d2h_overlap_frac"] <= 1.0
        # compute-stream busy time = union of the fp / bp / K2 intervals, within the step
        busy = sorted((e["start_ms"], e["end_ms"]) for e in trace if e["kind"] in ("fp", "bp", "k2_adamw"))
        union, cur = 0.0, None
        for a0, a1 in busy:
            if cur and a0 <= cur[1]:
                cur[1] = max(cur[1], a1)
            else:
                if cur:
                    union += cur[1] - cur[0]
                cur = [a0, a1]
        union += cur[1] - cur[0]
        assert 0 < st["compute_busy_ms"] <= st["last_step_ms"] + 1e-3
        assert abs(st["compute_busy_ms"] - union) <= 1e-3 * max(1.0, union)
    finally:
        tr.close()


def test_read_grad_after_landing_ring_reuse_is_an_error():
    tr, _, _ = engine_run(TINY, 1, 0, sh.SH_FP32, grad_ring_depth=1)
    try:
        # with a 1-deep landing ring only the last offloaded layer (layer 0 in BP order) survives
        g = tr.engine.read_layer(0, sh.SH_READ_GRAD)
        assert np.isfinite(g).all() and np.abs(g).max() > 0
        with pytest.raises(sh.ShError) as e:
            tr.engine.read_layer(TINY["L"] - 1, sh.SH_READ_GRAD)
        assert e.value.status == sh.SH_ERR_STATE
    finally:
        tr.close()


@pytest.mark.parametrize("precision,extra", [(sh.SH_BF16_MIXED, 0), (sh.SH_FP32, 0),
                                             (sh.SH_BF16_MIXED, sh.SH_FLAG_FETCH_FP32)])
def test_delay_injection_bitwise(precision, extra):
    """random host delays in the H2D/D2H issuers and the CPU Adam tasks perturb every
    cross-thread ordering; slot poisoning turns any read of a not-yet-arrived layer into NaNs.  The
    result must still equal the resident run bitwise (small landing ring, few threads)."""
    L = TINY["L"]
    ref, _, _ = engine_run(TINY, STEPS, L, precision)
    ref_state = engine_state(ref)
    ref.close()
    for w in (0, 1, 2):
        tr, _, _ = engine_run(TINY, STEPS, w, precision, cpu_threads=3, grad_ring_depth=2,
                              flags=sh.SH_FLAG_DELAY_INJECT | sh.SH_FLAG_POISON | extra)
        try:
            ok, what = states_bitwise_equal(engine_state(tr), ref_state)
            assert ok, (w, what)
        finally:
            tr.close()



@pytest.mark.parametrize("precision", [sh.SH_FP32, sh.SH_BF16_MIXED])
def test_ring_smaller_than_gpu_set_bitwise(precision):
    """R22: without clipping a GPU-optimised layer is updated right after its backward (per-layer
    K2), so the ring (prefetch distance + 1) may be smaller than the GPU-optimised set; its layers
    are then restaged by K1 from their HBM masters in FP as well.  Bitwise equal to resident."""
    L = TINY["L"]
    ref, _, _ = engine_run(TINY, STEPS, L, precision)
    ref_state = engine_state(ref)
    ref.close()
    for w, ring in ((3, 2), (L, 1), (L, 3), (2, 1)):
        tr, _, _ = engine_run(TINY, STEPS, w, precision, ring_slots=ring,
                              flags=sh.SH_FLAG_POISON | sh.SH_FLAG_DELAY_INJECT)
        try:
            ok, what = states_bitwise_equal(engine_state(tr), ref_state)
            assert ok, (w, ring, what)
            assert tr.engine.stats()["n_slots"] == min(ring, w + 1)
        finally:
            tr.close()
    # ring changes mid-run, together with the GPU-optimised set
    tr, _, _ = engine_run(TINY, 4, 1, precision, set_window_at={1: (3, 2), 2: (L, 1), 3: (0, 0)})
    try:
        ref2, _, _ = engine_run(TINY, 4, L, precision)
        ok, what = states_bitwise_equal(engine_state(tr), engine_state(ref2))
        ref2.close()
        assert ok, what
    finally:
        tr.close()


@pytest.mark.parametrize("precision,window", [(sh.SH_BF16_MIXED, 1), (sh.SH_FP32, 2)])
def test_checkpoint_resume_bitwise(precision, window):
    """Save after 2 steps (sh_read_layer: master, m, v of every layer and the resident set), restore
    into a fresh engine (sh_register_host_store with m, v and step=2, so Adam's bias correction
    continues at t=3) and train one more step: identical to an uninterrupted 3-step run."""
    from paper_conf_sc_sunwqyhxw22_b200 import trainer as T
    L = TINY["L"]
    full, _, _ = engine_run(TINY, 3, window, precision)
    want = engine_state(full)
    full.close()
    first, _, _ = engine_run(TINY, 2, window, precision)
    saved = {what: [first.read_layer_tensors(i, what) for i in range(L)] + [first.read_layer_tensors(-1, what)]
             for what in (sh.SH_READ_PARAM, sh.SH_READ_M, sh.SH_READ_V)}
    first.close()
    mc = T.ModelConfig(L, TINY["h"], TINY["nh"], TINY["s"], TINY["V"])
    tr = T.StrongholdTrainer(mc, batch=TINY["b"], window=window, precision=precision, init=False)
    try:
        p, m, v = saved[sh.SH_READ_PARAM], saved[sh.SH_READ_M], saved[sh.SH_READ_V]
        tr.register_state(p[:L], p[L], m[:L], v[:L], m[L], v[L], step=2)
        tr.set_tokens(synth.tokens(2, TINY["b"], TINY["s"], TINY["V"]))
        tr.step_device(want_norm=True)
        ok, what = states_bitwise_equal(engine_state(tr), want)
        assert ok, what
        assert tr.engine.stats()["step"] == 3
    finally:
        tr.close()
