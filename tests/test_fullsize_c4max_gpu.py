"""Parity at the size and in the launch configuration the DEFAULT `bench.py` times: c4max, BASELINE.json
configs[3] at "max trainable size per B200" -- h = 4096 GPT, L = 112 (22.8 B params, fp32 p/m/v 273 GB
> 180 GB of HBM), bf16 mixed, batch 16, the configuration the autotuner settles on (R27: 42
GPU-optimised layers, a decoupled ring of 26 slots; profiles/r02_ab_c4max_L112.txt), 8 host landing
buffers, the split host master (R25) and the lowest-computed-first offload order (R26).

The fp64 oracle cannot run this model, so (as test_fullsize_c4_gpu.py does for the 82-layer C4):
  * sampled AdamW at step 2 against the oracle's update, element by element, on a GPU-optimised layer
    (layer 0: its gradients are in the last-used GPU grad buffer), on every host layer whose gradients
    are still in one of the 8 landing buffers after the step (which ones depends on the offload
    timing: the step-1 state of every host layer is sampled) and on the resident set --
    the right gradients reach the right layer's GPU / CPU update at full size;
  * the split master at full size: the compute copy the engine hands out (SH_READ_COMPUTE) is the
    RNA bf16 of the fp32 master it reconstructs (SH_READ_PARAM), for a host layer and a GPU layer;
  * step-1 loss = ln V + h·0.02²/2 (Gaussian-logit closed form of the tied head at init).
"""
import math

import numpy as np
import pytest

import synth
from oracle import gpt_oracle as O
from tests._common import rna_bf16_bits

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

sh = pytest.importorskip("paper_conf_sc_sunwqyhxw22_b200.sh")
C4MAX = dict(L=112, h=4096, nh=32, s=1024, V=50304, b=16)
G_LAYERS, RING, LANDING = 42, 26, 8
HOST = tuple(range(G_LAYERS, 112))
SAMPLED = (0,) + HOST + (-1,)
N_SAMPLE = 4096


@pytest.fixture(scope="module")
def run():
    from paper_conf_sc_sunwqyhxw22_b200 import trainer as T
    rng = np.random.default_rng(1)
    h = C4MAX["h"]
    idx = {}
    for x in SAMPLED:
        n = sum(int(np.prod(s)) for s in (synth.layer_shapes(h) if x >= 0 else
                                          synth.resident_shapes(C4MAX["V"], C4MAX["s"], h)))
        idx[x] = np.sort(rng.choice(n, N_SAMPLE, replace=False))
    mc = T.ModelConfig(C4MAX["L"], h, C4MAX["nh"], C4MAX["s"], C4MAX["V"])
    tr = T.StrongholdTrainer(mc, batch=C4MAX["b"], window=G_LAYERS, ring_slots=RING, grad_ring_depth=LANDING,
                             precision=sh.SH_BF16_MIXED, flags=sh.SH_FLAG_PROFILE,
                             init_threads=16)
    out = {"loss": [], "s1": {}, "s2": {}}
    try:
        for t in range(2):
            tr.set_tokens(synth.tokens(t, C4MAX["b"], C4MAX["s"], C4MAX["V"]))
            tr.step_device()
            out["loss"].append(tr.loss())
            whats = (sh.SH_READ_PARAM, sh.SH_READ_M, sh.SH_READ_V)
            for x in SAMPLED:
                if t == 1:
                    try:
                        g = tr.engine.read_layer(x, sh.SH_READ_GRAD)[idx[x]]
                    except sh.ShError as e:  # a host layer's landing buffer was reused in this step
                        assert e.status == sh.SH_ERR_STATE and x in HOST, (x, e)
                        continue
                    out["s2"][x] = [tr.engine.read_layer(x, w)[idx[x]] for w in whats] + [g]
                else:
                    out["s1"][x] = [tr.engine.read_layer(x, w)[idx[x]] for w in whats]
        out["split"] = {x: (tr.engine.read_layer(x, sh.SH_READ_PARAM), tr.engine.read_layer(x, sh.SH_READ_COMPUTE))
                        for x in (0, G_LAYERS, C4MAX["L"] - 1)}
        out["stats"] = tr.engine.stats()
    finally:
        tr.close()
    return idx, out


def test_c4max_sampled_adamw_vs_oracle(run):
    idx, a = run
    st = a["stats"]
    assert st["window"] == G_LAYERS and st["landing_buffers"] == LANDING
    assert st["host_bytes"] >= 12 * (C4MAX["L"] - G_LAYERS) * 201_379_840  # the host store holds the rest
    opt = O.AdamWConfig()
    h = C4MAX["h"]
    checked = [x for x in SAMPLED if x in a["s2"]]
    assert 0 in checked and -1 in checked and any(x in checked for x in HOST), checked
    for x in checked:
        p1, m1, v1 = a["s1"][x]
        p2, m2, v2, g2 = a["s2"][x]
        numels = [int(np.prod(s)) for s in (synth.layer_shapes(h) if x >= 0 else
                                            synth.resident_shapes(C4MAX["V"], C4MAX["s"], h))]
        wd = synth.layer_weight_decay(h) if x >= 0 else synth.resident_weight_decay()
        decay = np.concatenate([np.full(n, d) for n, d in zip(numels, wd)])[idx[x]]
        assert np.abs(g2).max() > 0, x
        for d in (True, False):
            sel = decay == d
            if not sel.any():
                continue
            rp, rm, rv = O.adamw_update(p1[sel].astype(np.float64), g2[sel].astype(np.float64),
                                        m1[sel].astype(np.float64), v1[sel].astype(np.float64), 2, opt, d)
            scale = np.abs(p1[sel]) + np.abs(rp - p1[sel])
            assert (np.abs(p2[sel] - rp) <= 1e-6 * scale + 1e-30).all(), (x, d)
            mscale = opt.beta1 * np.abs(m1[sel]) + (1 - opt.beta1) * np.abs(g2[sel])
            assert (np.abs(m2[sel] - rm) <= 1e-6 * mscale + 1e-38).all(), (x, d)
            assert np.allclose(v2[sel], rv, rtol=1e-6, atol=1e-38), (x, d)


def test_c4max_compute_copy_is_rna_of_master(run):
    _, a = run
    for x, (p, c16) in a["split"].items():
        assert np.array_equal(c16, rna_bf16_bits(p)), x


def test_c4max_loss(run):
    _, a = run
    expect = math.log(C4MAX["V"]) + C4MAX["h"] * 0.02 ** 2 / 2
    assert abs(a["loss"][0] - expect) < 0.1, (a["loss"][0], expect)
    assert all(np.isfinite(a["loss"]))
