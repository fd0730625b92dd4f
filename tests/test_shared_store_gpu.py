"""Data-parallel shared host store with two real processes on the one GPU this
environment grants.  SH_FLAG_TEST_NO_COLLECTIVE replaces the NCCL average by the identity (both
ranks feed identical tokens, so the average IS the local gradient); everything else is the
production DP path: one /dev/shm store for both ranks, rank r offloads and CPU-updates only slice r
of every layer, prefetches wait on the cross-process per-layer counters.  The result must equal the
single-process run bitwise, on both ranks, for several windows."""
import os
import uuid

import numpy as np
import pytest
import torch.multiprocessing as mp

from tests._common import TINY, engine_run, engine_state, states_bitwise_equal

pytestmark = pytest.mark.gpu
sh = pytest.importorskip("paper_conf_sc_sunwqyhxw22_b200.sh")
STEPS = 3


def _rank(rank, world, name, window, q, extra_flags=0):
    import synth
    from paper_conf_sc_sunwqyhxw22_b200 import trainer as T
    os.environ["SH_WAIT_TIMEOUT_S"] = "120"
    mc = T.ModelConfig(TINY["L"], TINY["h"], TINY["nh"], TINY["s"], TINY["V"])
    tr = T.StrongholdTrainer(mc, batch=TINY["b"], window=window, precision=sh.SH_BF16_MIXED,
                             world_size=world, rank=rank, shm_name=name, cpu_threads=2, warmup_steps=2,
                             flags=sh.SH_FLAG_TEST_NO_COLLECTIVE | sh.SH_FLAG_CPU_HARD | extra_flags)
    for t in range(STEPS):
        tr.set_tokens(synth.tokens(t, TINY["b"], TINY["s"], TINY["V"]))
        tr.step_device()
    st = engine_state(tr)
    stats = tr.engine.stats()
    tr.close()
    q.put((rank, {k: [[a.tobytes() for a in u] if isinstance(u, list) else u.tobytes() for u in v]
                  for k, v in st.items()}, stats["d2h_bytes"], stats["window"]))


@pytest.mark.parametrize("window,extra", [(0, 0), (1, 0), (3, 0), (-1, 0), (1, "slice"), (0, "slice32")])
def test_shared_store_two_ranks_bitwise(window, extra):
    # window -1: both ranks autotune after 2 warm-up steps; rank 0's choice must be adopted by all
    ref, _, _ = engine_run(TINY, STEPS, window if window >= 0 else TINY["L"], sh.SH_BF16_MIXED)
    want = engine_state(ref)
    ref_d2h = ref.engine.stats()["d2h_bytes"]
    ref.close()
    want = {k: [[a.tobytes() for a in u] if isinstance(u, list) else u.tobytes() for u in v] for k, v in want.items()}
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    name = f"shtest_{uuid.uuid4().hex[:12]}"
    flags = {0: 0, "slice": sh.SH_FLAG_SLICE_FETCH,
             "slice32": sh.SH_FLAG_SLICE_FETCH | sh.SH_FLAG_FETCH_FP32}[extra]
    procs = [ctx.Process(target=_rank, args=(r, 2, name, window, q, flags)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(2)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    total_d2h = 0
    for rank, state, d2h, w in res:
        assert state == want, f"rank {rank} differs from the single-process run"
        total_d2h += d2h
    assert res[0][3] == res[1][3]  # same window on every rank
    if window >= 0:
        assert total_d2h == ref_d2h  # the two ranks together offload each host layer exactly once
    assert not any(f.startswith(name) for f in os.listdir("/dev/shm"))  # names removed after mapping
