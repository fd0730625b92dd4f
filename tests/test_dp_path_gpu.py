"""The data-parallel (collective) path of the engine on ONE GPU: SH_FLAG_TEST_DP_PATH builds a
one-rank NCCL communicator (ncclGetUniqueId / ncclCommInitRank through the dlopen'ed libnccl.so.2
torch loads), so every per-layer all-reduce and the resident-set
all-reduce are issued on the comm stream, ahead of K3, the gradient offload and the GPU-set K2,
exactly as with W > 1 -- and with one rank the average is the identity.

Bar: results bitwise equal to the single-GPU all-resident run for every window, in fp32, bf16 and
clip mode (the comm-stream ordering must not let K3 / D2H / K2 read a gradient before the
collective wrote it, nor a slot be refilled before they finished).
"""
import os

import pytest

from tests._common import TINY, engine_run, engine_state, states_bitwise_equal

# parity runs pin NCCL's algorithm and protocol: results must not depend on its tuner
os.environ.setdefault("NCCL_ALGO", "Ring")
os.environ.setdefault("NCCL_PROTO", "Simple")

pytestmark = pytest.mark.gpu

sh = pytest.importorskip("paper_conf_sc_sunwqyhxw22_b200.sh")

STEPS = 3


@pytest.mark.parametrize("precision,clip", [(sh.SH_FP32, 0.0), (sh.SH_BF16_MIXED, 0.0), (sh.SH_FP32, 0.5)])
def test_dp_path_one_rank_bitwise(precision, clip):
    L = TINY["L"]
    ref_tr, ref_losses, ref_norms = engine_run(TINY, STEPS, L, precision, max_grad_norm=clip)
    ref = engine_state(ref_tr)
    ref_tr.close()
    for w in (0, 1, 2, L):
        tr, losses, norms = engine_run(TINY, STEPS, w, precision, max_grad_norm=clip,
                                       flags=sh.SH_FLAG_TEST_DP_PATH, nccl_id=sh.nccl_unique_id())
        try:
            ok, what = states_bitwise_equal(engine_state(tr), ref)
            assert ok, f"window {w}: {what}"
            assert losses == ref_losses and norms == ref_norms
        finally:
            tr.close()


def test_dp_path_with_executors():
    """Executors (K4) feeding the collective path: K4 on the compute stream, then the all-reduce."""
    cfg = dict(TINY, b=4)
    ref_tr, ref_losses, _ = engine_run(cfg, STEPS, TINY["L"], sh.SH_FP32, executors=2)
    ref = engine_state(ref_tr)
    ref_tr.close()
    tr, losses, _ = engine_run(cfg, STEPS, 1, sh.SH_FP32, executors=2, flags=sh.SH_FLAG_TEST_DP_PATH,
                               nccl_id=sh.nccl_unique_id())
    try:
        ok, what = states_bitwise_equal(engine_state(tr), ref)
        assert ok, what
        assert losses == ref_losses
    finally:
        tr.close()


@pytest.mark.parametrize("fetch32", [False, True])
def test_dp_path_shared_store_slice_fetch_one_rank(fetch32):
    """The whole data-parallel machinery of one rank with real NCCL calls: the shared /dev/shm host
    store (control block, counters, barriers), NEXT-1 slice fetch (ncclCommSplit for the H2D issuer's
    communicator, in-place ncclAllGather after the slice H2D) and the per-layer all-reduce."""
    import os
    import uuid
    L = TINY["L"]
    ref_tr, ref_losses, _ = engine_run(TINY, STEPS, L, sh.SH_BF16_MIXED)
    ref = engine_state(ref_tr)
    ref_tr.close()
    name = f"shdp1_{uuid.uuid4().hex[:12]}"
    flags = sh.SH_FLAG_TEST_DP_PATH | sh.SH_FLAG_SLICE_FETCH | (sh.SH_FLAG_FETCH_FP32 if fetch32 else 0)
    tr, losses, _ = engine_run(TINY, STEPS, 1, sh.SH_BF16_MIXED, flags=flags, nccl_id=sh.nccl_unique_id(),
                               shm_name=name)
    try:
        ok, what = states_bitwise_equal(engine_state(tr), ref)
        assert ok, what
        assert losses == ref_losses
    finally:
        tr.close()
    assert not any(f.startswith(name) for f in os.listdir("/dev/shm"))
