"""Host-store footprint: only host-optimised layers hold a pinned host block (a layer joining the
GPU-optimised set gives its block back; one leaving it gets a new one), and the warm-up window of
an autotuned run (sh_config.warmup_window) decides which layers need a block from the start.
Footprint changes must not change a bit of the training."""
import pytest

import synth
from tests._common import TINY, engine_run, engine_state, states_bitwise_equal

pytestmark = pytest.mark.gpu

sh = pytest.importorskip("paper_conf_sc_sunwqyhxw22_b200.sh")


def test_blocks_follow_the_gpu_set():
    L = TINY["L"]
    ref_tr, ref_losses, _ = engine_run(TINY, 3, L, sh.SH_FP32)
    ref = engine_state(ref_tr)
    ref_tr.close()
    tr, losses, _ = engine_run(TINY, 1, 1, sh.SH_FP32)
    try:
        hb1 = tr.engine.stats()["host_bytes"]
        tr.engine.set_window(3)                      # layers 1, 2 join the GPU set
        hb3 = tr.engine.stats()["host_bytes"]
        assert hb3 < hb1
        per_layer = (hb1 - hb3) // 2
        assert per_layer >= 12 * sum(tr.mc.layer_numels())
        for t in (1, 2):
            if t == 2:
                tr.engine.set_window(1)              # and leave it again
                assert tr.engine.stats()["host_bytes"] == hb1
            tr.set_tokens(synth.tokens(t, TINY["b"], TINY["s"], TINY["V"]))
            tr.step_device(want_norm=True)
            losses.append(tr.loss())
        ok, what = states_bitwise_equal(engine_state(tr), ref)
        assert ok, what
        assert losses == ref_losses
    finally:
        tr.close()


def test_warmup_window_sets_the_initial_footprint():
    from paper_conf_sc_sunwqyhxw22_b200 import trainer as T
    mc = T.ModelConfig(TINY["L"], TINY["h"], TINY["nh"], TINY["s"], TINY["V"])
    a = T.StrongholdTrainer(mc, batch=TINY["b"], window=-1, precision=sh.SH_FP32, warmup_steps=2)
    b = T.StrongholdTrainer(mc, batch=TINY["b"], window=-1, precision=sh.SH_FP32, warmup_steps=2, warmup_window=3)
    try:
        sa, sb = a.engine.stats(), b.engine.stats()
        assert sa["window"] == 2 and sb["window"] == 3
        assert sb["host_bytes"] < sa["host_bytes"]
    finally:
        a.close()
        b.close()


def test_grow_landing_for_a_decoupled_ring():
    """SH_FLAG_GROW_LANDING: an autotune that decouples the ring (R22) grows a short landing ring to
    one buffer per host-optimised layer; the training stays bitwise equal to the resident run."""
    L = TINY["L"]
    ref_tr, ref_losses, _ = engine_run(TINY, 3, L, sh.SH_FP32)
    ref = engine_state(ref_tr)
    ref_tr.close()
    tr, losses, _ = engine_run(TINY, 1, 1, sh.SH_FP32, grad_ring_depth=1,
                               flags=sh.SH_FLAG_DECOUPLE | sh.SH_FLAG_GROW_LANDING)
    try:
        assert tr.engine.stats()["landing_buffers"] == 1
        # a profile whose solution is prefetch distance 1 (ring 2) and GPU set 2 (CPU-update bound)
        prof = dict(t_fp=[1.0] * L, t_bp=[3.0] * L, t_c2g=[0.1] * L, t_g2c=[0.1] * L, t_stage=[0.01] * L,
                    t_opt_gpu=[0.0] * L, t_opt_cpu=[8.0] * L, cpu_hard=True, cpu_util_max=1.0, decouple=True)
        assert sh.solve_window(**prof)["ring_slots"] == 2 and sh.solve_window(**prof)["window"] == 2
        assert tr.engine.autotune(prof) == 2
        st = tr.engine.stats()
        assert st["landing_buffers"] == L - 2 and st["n_slots"] >= 2
        for t in (1, 2):
            tr.set_tokens(synth.tokens(t, TINY["b"], TINY["s"], TINY["V"]))
            tr.step_device(want_norm=True)
            losses.append(tr.loss())
        ok, what = states_bitwise_equal(engine_state(tr), ref)
        assert ok, what
        assert losses == ref_losses
    finally:
        tr.close()


def test_late_shadow_bitwise():
    """SH_FLAG_LATE_SHADOW: fp32-fetch mode switches the host layers to bf16-shadow fetches after the
    autotune (shadow written from the master with the CPU Adam's RNE): bitwise the same training."""
    L = TINY["L"]
    ref_tr, ref_losses, _ = engine_run(TINY, 3, L, sh.SH_BF16_MIXED)
    ref = engine_state(ref_tr)
    ref_tr.close()
    tr, losses, _ = engine_run(TINY, 1, 1, sh.SH_BF16_MIXED, attention="flash",
                               flags=sh.SH_FLAG_FETCH_FP32 | sh.SH_FLAG_LATE_SHADOW | sh.SH_FLAG_GROW_LANDING,
                               grad_ring_depth=1)
    try:
        hb = tr.engine.stats()["host_bytes"]
        prof = dict(t_fp=[1.0] * L, t_bp=[3.0] * L, t_c2g=[0.1] * L, t_g2c=[0.1] * L, t_stage=[0.01] * L,
                    t_opt_gpu=[0.0] * L, t_opt_cpu=[8.0] * L, cpu_hard=True, cpu_util_max=1.0, decouple=True)
        assert tr.engine.autotune(prof) == 2
        st = tr.engine.stats()
        assert st["landing_buffers"] == L - 2
        h2d0 = st["h2d_bytes"]
        for t in (1, 2):
            tr.set_tokens(synth.tokens(t, TINY["b"], TINY["s"], TINY["V"]))
            tr.step_device(want_norm=True)
            losses.append(tr.loss())
        # host layers now fetch 2 B/param (bf16 shadow), not 4
        per_fetch = (tr.engine.stats()["h2d_bytes"] - h2d0) / max(1, tr.engine.stats()["h2d_copies"] - st["h2d_copies"])
        assert per_fetch <= 2 * sum(tr.mc.layer_numels()) * 1.01
        ok, what = states_bitwise_equal(engine_state(tr), ref)
        assert ok, what
        assert losses == ref_losses
    finally:
        tr.close()


@pytest.mark.parametrize("policy", ["SH_NUMA_SPLIT", "SH_NUMA_LOCAL", "SH_NUMA_INTERLEAVE"])
def test_numa_placement_bitwise(tmp_path, monkeypatch, policy):
    """NUMA placement on a fake two-node topology that splits the box's real
    CPUs: workers are pinned to their half, SPLIT workers prefer their node's layers, blocks are
    mbind'ed (node 0 exists, the fake node 1 does not, so only its binds fail).  Placement and
    job routing must not change a bit of the training."""
    import os
    n = os.cpu_count()
    if n < 2:
        pytest.skip("needs 2 CPUs")
    root = tmp_path / "sysfs"
    base = root / "sys/devices/system/node"
    base.mkdir(parents=True)
    (base / "online").write_text("0-1\n")
    for k, cl in enumerate((f"0-{n // 2 - 1}", f"{n // 2}-{n - 1}")):
        (base / f"node{k}").mkdir()
        (base / f"node{k}" / "cpulist").write_text(cl + "\n")
    L = TINY["L"]
    ref_tr, ref_losses, _ = engine_run(TINY, 3, L, sh.SH_FP32)
    ref = engine_state(ref_tr)
    ref_tr.close()
    monkeypatch.setenv("SH_SYSFS_ROOT", str(root))
    assert len(sh.numa_topology()) == 2  # refresh the library's cached topology
    try:
        pol = getattr(sh, policy)
        tr, losses, _ = engine_run(TINY, 3, 1, sh.SH_FP32, cpu_threads=4, numa_policy=pol)
        try:
            st = tr.engine.stats()
            assert st["numa_nodes"] == 2 and st["numa_policy"] == pol
            if pol == sh.SH_NUMA_INTERLEAVE:
                assert st["numa_pinned_workers"] == 0
            else:
                assert st["numa_pinned_workers"] == 4
            if pol == sh.SH_NUMA_SPLIT:
                assert st["numa_bound_bytes"] > 0  # the node-0 layers
            ok, what = states_bitwise_equal(engine_state(tr), ref)
            assert ok, what
            assert losses == ref_losses
        finally:
            tr.close()
    finally:
        monkeypatch.delenv("SH_SYSFS_ROOT")
        sh.numa_topology()
