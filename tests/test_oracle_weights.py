"""Pins for the O4 weight generator (oracle/weights.py) -- CPU only."""
import math

import numpy as np
import torch

from oracle.weights import Weights, bf16_rne, gen, scale_for, splitmix64
from workloads.configs import MODELS


def test_splitmix64_published_vectors():
    # Vigna's splitmix64 reference: seed 1234567 -> 6457827717110365317, 3203168211198807973, ...
    g = 0x9E3779B97F4A7C15
    seeds = np.array([1234567, (1234567 + g) % 2 ** 64, (1234567 + 2 * g) % 2 ** 64], dtype=np.uint64)
    out = [int(v) for v in splitmix64(seeds)]
    assert out == [6457827717110365317, 3203168211198807973, 9817491932198370423]
    assert int(splitmix64(np.array([0], np.uint64))[0]) == 0xE220A8397B1DCDAF


def test_bf16_rne_matches_torch_cast():
    rng = np.random.default_rng(0)
    f = np.concatenate([rng.standard_normal(100000).astype(np.float32) * 3,
                        # exact ties: mantissa low half == 0x8000, both parities
                        (np.arange(1, 2000, dtype=np.uint32) << 16 | 0x8000).view(np.float32)])
    ref = torch.from_numpy(f).to(torch.bfloat16).to(torch.float32).numpy()
    assert np.array_equal(bf16_rne(f), ref)


def test_generator_range_moments_and_bf16_exactness():
    s = scale_for("proj", 4096)
    w = gen(1001, 5, 1 << 20, s)
    assert np.all(np.abs(w) <= np.float32(s) * 1.0079)          # |x| <= 1, one bf16 rounding up
    sigma = 1.0 / math.sqrt(4096)
    assert abs(w.std() / sigma - 1.0) < 0.01
    assert abs(w.mean()) < 3 * sigma / math.sqrt(w.size) * 3
    assert np.array_equal(bf16_rne(w), w)                          # already bf16 values
    # x = (u - 2^23) 2^-23 is exact in fp32; distinct tensors / seeds decorrelate
    w2 = gen(1001, 6, 1 << 20, s)
    assert abs(np.corrcoef(w, w2)[0, 1]) < 0.01
    # streaming in pieces equals one shot (counter-based)
    assert np.array_equal(gen(1001, 5, 1000, s, start=5000), w[5000:6000])


def test_embedding_rows_match_full_table():
    m = MODELS["C0"]
    W = Weights(m)
    full = gen(m.weight_seed, 0xFFFFF0, m.vocab * m.hidden, scale_for("embed")).reshape(m.vocab, m.hidden)
    ids = np.array([3, 511, 3, 0, 17])
    assert np.array_equal(W.embed_rows(ids), full[ids])
