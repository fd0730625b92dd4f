"""Data-parallel host-side logic with world_size 2 on CPU (gloo), no GPU.

(The engine itself at world_size 2 -- sh_init(world_size=2) in two processes bootstrapped with gloo,
different data per rank, the collectives through a shared host segment, parity with the oracle's
global batch -- is tests/test_dp_host_gpu.py; sh_init needs a CUDA device.)

On a B200 box each rank averages a layer's gradients with ncclAllReduce(avg) before the offload
 and its CPU AdamW pool updates its replica of the host store.  Here the
collective is gloo and the update is the same native CPU AdamW (sh_op_adamw_cpu): the test pins
(a) every rank ends with bitwise-identical parameters/moments/shadows, (b) they equal a single
process updating with the global-batch mean gradient, (c) the nccl-unique-id broadcast path
delivers rank 0's 128 bytes to every rank (the bootstrap bench.py uses).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import synth

sh = pytest.importorskip("paper_conf_sc_sunwqyhxw22_b200.sh")

N = 1 << 14
ND = 1 << 13


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    # bootstrap: rank 0's id reaches everyone
    idt = torch.zeros(128, dtype=torch.uint8)
    if rank == 0:
        idt.copy_(torch.arange(128, dtype=torch.uint8))
    dist.broadcast(idt, 0)
    ok_id = bool((idt == torch.arange(128, dtype=torch.uint8)).all())
    p, _, m, v = synth.random_adam_state(7, N)
    results = []
    for step in range(1, 4):
        g_local = synth.normal(synth.stream_key(100 + step, rank), N, 1e-3)
        g = torch.from_numpy(g_local.copy())
        dist.all_reduce(g, op=dist.ReduceOp.SUM)
        g_avg = (g.numpy() * np.float32(1.0 / world)).astype(np.float32)
        sc = sh.adam_scalars(1e-3, 0.9, 0.999, 1e-8, 0.01, step)
        shadow = np.empty(N, np.uint16)
        sh.op_adamw_cpu(p, m, v, g_avg, shadow, N, ND, sc, threads=2)
        results.append((p.copy(), m.copy(), v.copy(), shadow.copy()))
    gathered = [None] * world
    dist.all_gather_object(gathered, [tuple(a.tobytes() for a in r) for r in results])
    if rank == 0:
        out.put((ok_id, gathered))
    dist.destroy_process_group()


def test_dp_ranks_bitwise_identical_and_equal_global_mean():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    ok_id, gathered = q.get(timeout=120)
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    assert ok_id
    assert gathered[0] == gathered[1]  # (a) identical on every rank
    # (b) single process with the global-batch mean gradient
    p, _, m, v = synth.random_adam_state(7, N)
    for step in range(1, 4):
        gs = [synth.normal(synth.stream_key(100 + step, r), N, 1e-3) for r in range(world)]
        g_avg = ((gs[0] + gs[1]) * np.float32(0.5)).astype(np.float32)
        sc = sh.adam_scalars(1e-3, 0.9, 0.999, 1e-8, 0.01, step)
        shadow = np.empty(N, np.uint16)
        sh.op_adamw_cpu(p, m, v, g_avg, shadow, N, ND, sc, threads=1)
        assert (p.tobytes(), m.tobytes(), v.tobytes(), shadow.tobytes()) == gathered[0][step - 1]
