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


def test_warm_kv_index_layout_and_counter_property():
    # O4 warm start: element ((r*2^17 + p)*Hkv + h)*D + j of tensor 0xEE0000 + 2l (+1 V)
    from oracle.weights import T_WARM_K, warm_kv
    seed, Hkv, D = 1004, 8, 128
    k, v = warm_kv(seed, 5, 40, 3, Hkv, D)
    assert k.shape == (40, Hkv, D) and v.shape == (40, Hkv, D)
    # a longer context extends the same values (counter-based: position p never depends on the length)
    k2, v2 = warm_kv(seed, 5, 100, 3, Hkv, D)
    assert np.array_equal(k2[:40], k) and np.array_equal(v2[:40], v)
    # element (p=17, h=6, j=99) is counter (5*2^17 + 17)*1024 + 6*128 + 99 of the layer's K tensor
    i = (5 * 2 ** 17 + 17) * Hkv * D + 6 * D + 99
    assert k[17, 6, 99] == gen(seed, T_WARM_K + 6, 1, scale_for("embed"), start=i)[0]
    assert v[17, 6, 99] == gen(seed, T_WARM_K + 7, 1, scale_for("embed"), start=i)[0]
    # different request / layer / K vs V streams are decorrelated; sigma = 1, bf16 exact
    kk, _ = warm_kv(seed, 6, 40, 3, Hkv, D)
    kl, _ = warm_kv(seed, 5, 40, 4, Hkv, D)
    for a, b in ((k, kk), (k, kl), (k, v)):
        assert abs(np.corrcoef(a.ravel(), b.ravel())[0, 1]) < 0.02
    assert abs(k.std() - 1.0) < 0.02 and np.array_equal(bf16_rne(k), k)


def test_threaded_generation_equals_one_shot():
    from oracle.weights import gen_threads
    s = scale_for("proj", 512)
    assert np.array_equal(gen_threads(7, 9, 3_000_001, s, start=11, chunk=1 << 18), gen(7, 9, 3_000_001, s, start=11))
