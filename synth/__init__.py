"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

This module holds NO arithmetic of the method (no forward, backward, norm or
optimizer math).  It only turns (seed, tag) into numbers with a counter-based
generator, so that both sides of every parity test start from identical fp32
parameters and int32 tokens.

Recipe (SURVEY.md §8(c) reading #14, §8(d) Inputs):
  * generator: splitmix64(seed, tag, counter) -> uniform (0,1) via the top 53 bits.
  * weights 2-D: N(0, 0.02) by Box-Muller; residual output projections
    (W_o, W_proj) N(0, 0.02/sqrt(2L)) (GPT-2 init);  biases 0; LN gamma 1, beta 0.
  * embedding E [V,h] and learned positions Pos [s,h]: N(0, 0.02).
  * tokens: uniform integers in [0, V), one stream per step: seed 1234 + step.
The paper (§V-B) only says "GPT-like Transformer-based models";
the GPT-2 pre-LN structure and this init are the readings listed in DESIGN.md.
"""
from __future__ import annotations

import numpy as np

_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def _mix(z: np.ndarray) -> np.ndarray:
    z = (z ^ (z >> np.uint64(30))) * _M1
    z = (z ^ (z >> np.uint64(27))) * _M2
    return z ^ (z >> np.uint64(31))


def stream_key(seed: int, *tags: int) -> np.uint64:
    """Derive a 64-bit stream key from a seed and integer tags (splitmix64 chaining)."""
    with np.errstate(over="ignore"):
        k = np.uint64(seed & 0xFFFFFFFFFFFFFFFF)
        for t in tags:
            k = _mix(np.array([k + _GOLDEN * np.uint64((t + 1) & 0xFFFFFFFFFFFFFFFF)], dtype=np.uint64))[0]
    return k


def uniform_u64(key: np.uint64, n: int, offset: int = 0) -> np.ndarray:
    """n raw 64-bit outputs of splitmix64 at counters offset+1 .. offset+n for stream `key`."""
    with np.errstate(over="ignore"):
        ctr = np.arange(offset + 1, offset + n + 1, dtype=np.uint64)
        return _mix(key + ctr * _GOLDEN)


def uniform01(key: np.uint64, n: int, offset: int = 0) -> np.ndarray:
    """Uniform doubles in the open interval (0, 1)."""
    u = uniform_u64(key, n, offset) >> np.uint64(11)
    return (u.astype(np.float64) + 0.5) * (1.0 / 9007199254740992.0)


def normal(key: np.uint64, n: int, std: float) -> np.ndarray:
    """N(0, std) as float32 via Box-Muller on pairs of uniforms (fp64 math, rounded once)."""
    m = (n + 1) // 2
    u1 = uniform01(key, m, 0)
    u2 = uniform01(key, m, m)
    r = np.sqrt(-2.0 * np.log(u1))
    z = np.empty(2 * m, dtype=np.float64)
    z[0::2] = r * np.cos(2.0 * np.pi * u2)
    z[1::2] = r * np.sin(2.0 * np.pi * u2)
    return (z[:n] * std).astype(np.float32)


def fill_normal(out: np.ndarray, key: np.uint64, std: float, threads: int = 8, chunk_pairs: int = 1 << 20):
    """Write normal(key, out.size, std) into the float32 array `out` (bit-identical to normal()),
    in chunks of Box-Muller pairs on `threads` threads, with O(chunk) temporary memory."""
    from concurrent.futures import ThreadPoolExecutor
    n = out.size
    m = (n + 1) // 2
    flat = out.reshape(-1)

    def work(k0):
        k1 = min(m, k0 + chunk_pairs)
        u1 = uniform01(key, k1 - k0, k0)
        u2 = uniform01(key, k1 - k0, m + k0)
        r = np.sqrt(-2.0 * np.log(u1))
        z0 = ((r * np.cos(2.0 * np.pi * u2)) * std).astype(np.float32)
        z1 = ((r * np.sin(2.0 * np.pi * u2)) * std).astype(np.float32)
        e0 = 2 * k1 if 2 * k1 <= n else n
        flat[2 * k0:e0:2] = z0[: (e0 - 2 * k0 + 1) // 2]
        flat[2 * k0 + 1:min(2 * k1, n):2] = z1[: (min(2 * k1, n) - 2 * k0) // 2]

    with ThreadPoolExecutor(max(1, threads)) as ex:
        list(ex.map(work, range(0, m, chunk_pairs)))
    return out


# --- GPT-2 shaped parameter sets -------------------------------------------------

LAYER_TENSORS = ("ln1_g", "ln1_b", "w_qkv", "b_qkv", "w_o", "b_o",
                 "ln2_g", "ln2_b", "w_fc", "b_fc", "w_proj", "b_proj")
RESIDENT_TENSORS = ("wte", "wpe", "lnf_g", "lnf_b")


def layer_shapes(h: int) -> list[tuple[int, ...]]:
    """Tensor shapes of one transformer block in the packed order."""
    return [(h,), (h,), (3 * h, h), (3 * h,), (h, h), (h,),
            (h,), (h,), (4 * h, h), (4 * h,), (h, 4 * h), (h,)]


def layer_weight_decay(h: int) -> list[bool]:
    """Decoupled weight decay applies to 2-D weights only (Megatron convention, reading #2)."""
    return [len(s) == 2 for s in layer_shapes(h)]


def resident_shapes(V: int, s: int, h: int) -> list[tuple[int, ...]]:
    return [(V, h), (s, h), (h,), (h,)]


def resident_weight_decay() -> list[bool]:
    return [True, True, False, False]


def init_layer(seed: int, layer: int, L: int, h: int) -> list[np.ndarray]:
    """fp32 initial tensors of block `layer` (list in LAYER_TENSORS order)."""
    out = []
    resid_std = 0.02 / np.sqrt(2.0 * L)
    for ti, (name, shp) in enumerate(zip(LAYER_TENSORS, layer_shapes(h))):
        n = int(np.prod(shp))
        if name.startswith("w_"):
            std = resid_std if name in ("w_o", "w_proj") else 0.02
            out.append(normal(stream_key(seed, 1, layer, ti), n, std).reshape(shp))
        elif name.endswith("_g"):
            out.append(np.ones(shp, dtype=np.float32))
        else:
            out.append(np.zeros(shp, dtype=np.float32))
    return out


def init_layer_into(flat: np.ndarray, seed: int, layer: int, L: int, h: int, threads: int = 8) -> np.ndarray:
    """init_layer(...) concatenated in LAYER_TENSORS order, written into the float32 vector
    `flat` (bit-identical, bounded temporaries; used for multi-billion-parameter configs)."""
    resid_std = 0.02 / np.sqrt(2.0 * L)
    o = 0
    for ti, (name, shp) in enumerate(zip(LAYER_TENSORS, layer_shapes(h))):
        n = int(np.prod(shp))
        seg = flat[o:o + n]
        if name.startswith("w_"):
            std = resid_std if name in ("w_o", "w_proj") else 0.02
            fill_normal(seg, stream_key(seed, 1, layer, ti), std, threads)
        elif name.endswith("_g"):
            seg[:] = 1.0
        else:
            seg[:] = 0.0
        o += n
    return flat


def init_resident_into(flat: np.ndarray, seed: int, V: int, s: int, h: int, threads: int = 8) -> np.ndarray:
    fill_normal(flat[:V * h], stream_key(seed, 2, 0), 0.02, threads)
    fill_normal(flat[V * h:V * h + s * h], stream_key(seed, 2, 1), 0.02, threads)
    flat[V * h + s * h:V * h + s * h + h] = 1.0
    flat[V * h + s * h + h:] = 0.0
    return flat


def init_resident(seed: int, V: int, s: int, h: int) -> list[np.ndarray]:
    wte = normal(stream_key(seed, 2, 0), V * h, 0.02).reshape(V, h)
    wpe = normal(stream_key(seed, 2, 1), s * h, 0.02).reshape(s, h)
    return [wte, wpe, np.ones(h, np.float32), np.zeros(h, np.float32)]


def tokens(step: int, n_seq: int, s: int, V: int, base_seed: int = 1234) -> np.ndarray:
    """int32 [n_seq, s+1] uniform token ids for `step` (inputs = [:, :s], targets = [:, 1:])."""
    key = stream_key(base_seed + step, 3)
    u = uniform_u64(key, n_seq * (s + 1))
    return (u % np.uint64(V)).astype(np.int32).reshape(n_seq, s + 1)


def random_adam_state(seed: int, n: int, scale_p=0.05, scale_g=1e-3):
    """Random fp32 (p, g, m, v) arrays for optimizer-only parity tests (v >= 0)."""
    p = normal(stream_key(seed, 4, 0), n, scale_p)
    g = normal(stream_key(seed, 4, 1), n, scale_g)
    m = normal(stream_key(seed, 4, 2), n, scale_g)
    v = np.abs(normal(stream_key(seed, 4, 3), n, scale_g)) ** 2
    return p, g, m, v.astype(np.float32)
