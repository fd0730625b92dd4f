"""The seeded generator: chunked/threaded fills are bit-identical to the reference form, and
the draws have the intended distribution (no method arithmetic lives in synth/)."""
import numpy as np

import synth


def test_fill_normal_bit_identical_to_normal():
    key = synth.stream_key(3, 1, 2)
    for n in (1, 2, 7, 1000, (1 << 16) + 3):
        ref = synth.normal(key, n, 0.02)
        for chunk in (1, 3, 1 << 10, 1 << 20):
            out = np.empty(n, np.float32)
            synth.fill_normal(out, key, 0.02, threads=3, chunk_pairs=chunk)
            assert out.tobytes() == ref.tobytes(), (n, chunk)


def test_init_layer_into_matches_init_layer():
    L, h = 3, 64
    for layer in range(L):
        ref = np.concatenate([a.reshape(-1) for a in synth.init_layer(9, layer, L, h)])
        out = np.full(ref.size, np.nan, np.float32)
        synth.init_layer_into(out, 9, layer, L, h, threads=2)
        assert out.tobytes() == ref.tobytes()
    ref = np.concatenate([a.reshape(-1) for a in synth.init_resident(9, 40, 16, h)])
    out = np.full(ref.size, np.nan, np.float32)
    synth.init_resident_into(out, 9, 40, 16, h, threads=2)
    assert out.tobytes() == ref.tobytes()


def test_normal_moments_and_tokens_range():
    z = synth.normal(synth.stream_key(1), 1 << 20, 1.0).astype(np.float64)
    assert abs(z.mean()) < 5e-3 and abs(z.std() - 1.0) < 5e-3
    assert abs((z ** 4).mean() - 3.0) < 3e-2  # Gaussian kurtosis
    t = synth.tokens(0, 4, 1023, 50304)
    assert t.shape == (4, 1024) and t.min() >= 0 and t.max() < 50304
    counts = np.bincount(synth.tokens(1, 64, 1023, 16).reshape(-1), minlength=16)
    assert counts.min() > 0.8 * counts.mean()
