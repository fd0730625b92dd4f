"""NEXT-2 secondary-storage tier: host-optimised layers kept in files under
sh_config.spill_dir instead of pinned host RAM, read and written with O_DIRECT bulk requests
(io_uring) through pinned bounce / staging buffers.

Bar: moving a layer's master / m / v (/ bf16 shadow) to a file must not change a single bit --
the windowed run with spilled layers equals the all-resident run bitwise (the same invariant as
every other window), in fp32, bf16-shadow and fp32-fetch modes, and after a window change that
moves layers between the GPU set and the spill tier.
"""
import os

import pytest

from tests._common import TINY, engine_run, engine_state, states_bitwise_equal

pytestmark = pytest.mark.gpu

sh = pytest.importorskip("paper_conf_sc_sunwqyhxw22_b200.sh")

STEPS = 3


@pytest.fixture(scope="module")
def resident():
    out = {}
    for prec in (sh.SH_FP32, sh.SH_BF16_MIXED):
        tr, losses, norms = engine_run(TINY, STEPS, TINY["L"], prec)
        out[prec] = (engine_state(tr), losses, norms)
        tr.close()
    return out


@pytest.mark.parametrize("precision,flags", [(sh.SH_FP32, 0), (sh.SH_BF16_MIXED, 0),
                                             (sh.SH_BF16_MIXED, sh.SH_FLAG_FETCH_FP32),
                                             (sh.SH_FP32, sh.SH_FLAG_SPILL_EVICT)])
@pytest.mark.parametrize("window", [0, 1])
def test_spilled_bitwise_equals_resident(tmp_path, resident, precision, flags, window):
    ref, ref_losses, ref_norms = resident[precision]
    tr, losses, norms = engine_run(TINY, STEPS, window, precision, flags=flags, spill_dir=str(tmp_path),
                                   host_pin_budget_bytes=1)  # every host-optimised layer spills
    try:
        st = tr.engine.stats()
        assert st["spilled_layers"] == TINY["L"] - window and st["spill_bytes"] > 0
        # every step reads each spilled layer's fetch region(s) and its master / m / v, and writes them back
        assert st["spill_read_bytes"] > 0 and st["spill_write_bytes"] > 0 and st["spill_io_ms"] > 0
        ok, what = states_bitwise_equal(engine_state(tr), ref)
        assert ok, what
        assert losses == ref_losses and norms == ref_norms
        assert os.listdir(tmp_path) == []  # the files are unlinked at creation
    finally:
        tr.close()


def test_partial_spill_and_window_change(tmp_path, resident):
    ref, ref_losses, _ = resident[sh.SH_FP32]
    # a budget that pins the landing ring and one layer block; the remaining host layers spill
    probe, _, _ = engine_run(TINY, 1, TINY["L"] - 1, sh.SH_FP32)
    one_layer = probe.engine.stats()["host_bytes"]
    probe.close()
    tr, losses, _ = engine_run(TINY, STEPS, 1, sh.SH_FP32, spill_dir=str(tmp_path), host_pin_budget_bytes=one_layer,
                               set_window_at={1: 3, 2: 2})  # spilled layers move into HBM and back
    try:
        st = tr.engine.stats()
        assert 0 < st["spilled_layers"] < TINY["L"] - 1
        ok, what = states_bitwise_equal(engine_state(tr), ref)
        assert ok, what
        assert losses == ref_losses
    finally:
        tr.close()


def test_bad_spill_dir(tmp_path):
    with pytest.raises(sh.ShError):
        tr, _, _ = engine_run(TINY, 1, 1, sh.SH_FP32, spill_dir=str(tmp_path / "missing"))
        tr.close()


def test_spill_clip_mode_bitwise(tmp_path):
    L = TINY["L"]
    ref_tr, ref_losses, ref_norms = engine_run(TINY, STEPS, L, sh.SH_FP32, max_grad_norm=0.5)
    ref = engine_state(ref_tr)
    ref_tr.close()
    tr, losses, norms = engine_run(TINY, STEPS, 1, sh.SH_FP32, max_grad_norm=0.5, spill_dir=str(tmp_path),
                                   host_pin_budget_bytes=1)
    try:
        assert tr.engine.stats()["spilled_layers"] == L - 1
        ok, what = states_bitwise_equal(engine_state(tr), ref)
        assert ok, what
        assert losses == ref_losses and norms == ref_norms
    finally:
        tr.close()
