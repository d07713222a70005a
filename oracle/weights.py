"""ORACLE (test infrastructure only) -- counter-based weight generator O4 (numpy).

Spec (the paper loads random "dummy"
weights for its own runs):

    u  = splitmix64(seed ^ (t << 40) ^ i) >> 40          (24 bits)
    x  = (u - 2^23) * 2^-23                               (exact fp32, in [-1, 1))
    s_t = fp32(sqrt(3 / fan_in))  (projections),  fp32(sqrt(3) * 0.02) (biases),
          fp32(sqrt(3)) (embedding), fp32(sqrt(3 / H)) (LM head)
    w  = bf16_rne(fp32(x * s_t))                          (one rounded fp32 multiply, then RNE)

so w is uniform with std sigma_t.  Norm gains are exactly 1.  Tensor ids:
t = 1 + 16*layer + kind (kind: 0 Wq, 1 Wk, 2 Wv, 3 Wo, 4 Wgate, 5 Wup, 6 Wdown,
7 bq, 8 bk, 9 bv); embedding t = 0xFFFFF0, LM head t = 0xFFFFF1.  i is the
row-major index in the logical [out_features, in_features] matrix.

This module is an independent implementation of the generator; the CUDA init
kernel implements the same spec on its own (no shared code).
Pinned by: tests/test_oracle_weights.py (splitmix64 published test vector,
exact-range / moment checks, bf16 RNE against torch's own bf16 cast).
"""
from __future__ import annotations

import math

import numpy as np

M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
KIND = dict(wq=0, wk=1, wv=2, wo=3, wg=4, wu=5, wd=6, bq=7, bk=8, bv=9)
T_EMBED = 0xFFFFF0
T_LMHEAD = 0xFFFFF1


def splitmix64(x: np.ndarray) -> np.ndarray:
    """Vigna's splitmix64 finaliser applied to state x (uint64 wrap-around)."""
    x = x.astype(np.uint64, copy=True)
    x += np.uint64(0x9E3779B97F4A7C15)
    z = x
    z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
    z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
    return z ^ (z >> np.uint64(31))


def bf16_rne(f: np.ndarray) -> np.ndarray:
    """Round fp32 to the nearest bf16 (ties to even); returned as fp32 holding the bf16 value."""
    u = np.ascontiguousarray(f, dtype=np.float32).view(np.uint32).astype(np.uint64)
    u = (u + np.uint64(0x7FFF) + ((u >> np.uint64(16)) & np.uint64(1))) & np.uint64(0xFFFF0000)
    return u.astype(np.uint32).view(np.float32)


def scale_for(sigma_kind: str, fan_in: int = 0) -> np.float32:
    if sigma_kind == "proj":
        return np.float32(math.sqrt(3.0 / fan_in))
    if sigma_kind == "bias":
        return np.float32(math.sqrt(3.0) * 0.02)
    if sigma_kind == "embed":
        return np.float32(math.sqrt(3.0))
    raise ValueError(sigma_kind)


def gen(seed: int, t: int, n: int, scale: np.float32, start: int = 0) -> np.ndarray:
    """Elements [start, start+n) of tensor t, as fp32 holding exact bf16 values."""
    i = np.arange(start, start + n, dtype=np.uint64)
    key = np.uint64(seed) ^ (np.uint64(t) << np.uint64(40))
    u = splitmix64(key ^ i) >> np.uint64(40)
    x = ((u.astype(np.int64) - (1 << 23)).astype(np.float32)) * np.float32(2.0 ** -23)
    return bf16_rne(x * np.float32(scale))


# Warm-start KV (SURVEY.md §8(c) O4 last item; C4's warm decode set, §8(d)): K and V of warm request r at
# position p, layer l, kv head h, dim j are element i = ((r * 2^17 + p) * Hkv + h) * D + j of tensor
# T_WARM_K + 2 l (K) / T_WARM_K + 2 l + 1 (V), scale sqrt(3) (sigma 1, the size of a RoPE'd k of a
# unit-rms input under 1/sqrt(H) weights).  Needs p < 2^17 and (r * 2^17 + p) * Hkv * D < 2^40.
T_WARM_K = 0xEE0000
WARM_POS_BITS = 17


def warm_kv(seed: int, req_id: int, context_len: int, layer: int, n_kv_heads: int, head_dim: int):
    """(K, V) [context_len, n_kv_heads, head_dim] of a warm sequence at one layer (fp32 holding bf16)."""
    assert context_len <= (1 << WARM_POS_BITS)
    per_pos = n_kv_heads * head_dim
    start = (req_id << WARM_POS_BITS) * per_pos
    assert start + context_len * per_pos <= (1 << 40)
    s = scale_for("embed")
    k = gen(seed, T_WARM_K + 2 * layer, context_len * per_pos, s, start)
    v = gen(seed, T_WARM_K + 2 * layer + 1, context_len * per_pos, s, start)
    return k.reshape(context_len, n_kv_heads, head_dim), v.reshape(context_len, n_kv_heads, head_dim)


def gen_threads(seed: int, t: int, n: int, scale: np.float32, start: int = 0, chunk: int = 1 << 22) -> np.ndarray:
    """`gen` over [start, start+n) in independent chunks on a thread pool (numpy releases the GIL in
    its ufuncs); element for element identical to one `gen` call (counter-based)."""
    if n <= chunk:
        return gen(seed, t, n, scale, start)
    from concurrent.futures import ThreadPoolExecutor
    out = np.empty(n, np.float32)

    def one(o):
        m = min(chunk, n - o)
        out[o:o + m] = gen(seed, t, m, scale, start + o)
    with ThreadPoolExecutor() as ex:
        list(ex.map(one, range(0, n, chunk)))
    return out


def layer_tid(layer: int, kind: str) -> int:
    return 1 + 16 * layer + KIND[kind]


class Weights:
    """Lazily generated oracle weights for one ModelShape (fp32 arrays holding bf16 values)."""

    def __init__(self, m, dtype=np.float32):
        self.m = m
        self.dtype = dtype
        self._cache = {}

    def _mat(self, t, rows, cols, scale):
        key = (t, rows, cols)
        if key not in self._cache:
            self._cache[key] = gen_threads(self.m.weight_seed, t, rows * cols, scale).reshape(rows, cols).astype(self.dtype)
        return self._cache[key]

    def layer(self, l: int) -> dict:
        m = self.m
        H, qd, kd, I = m.hidden, m.q_dim, m.kv_dim, m.intermediate
        w = dict(
            wq=self._mat(layer_tid(l, "wq"), qd, H, scale_for("proj", H)),
            wk=self._mat(layer_tid(l, "wk"), kd, H, scale_for("proj", H)),
            wv=self._mat(layer_tid(l, "wv"), kd, H, scale_for("proj", H)),
            wo=self._mat(layer_tid(l, "wo"), H, qd, scale_for("proj", qd)),
            wg=self._mat(layer_tid(l, "wg"), I, H, scale_for("proj", H)),
            wu=self._mat(layer_tid(l, "wu"), I, H, scale_for("proj", H)),
            wd=self._mat(layer_tid(l, "wd"), H, I, scale_for("proj", I)),
            g1=np.ones(H, self.dtype), g2=np.ones(H, self.dtype),
        )
        if m.qkv_bias:
            w["bq"] = self._mat(layer_tid(l, "bq"), 1, qd, scale_for("bias"))[0]
            w["bk"] = self._mat(layer_tid(l, "bk"), 1, kd, scale_for("bias"))[0]
            w["bv"] = self._mat(layer_tid(l, "bv"), 1, kd, scale_for("bias"))[0]
        return w

    def embed_rows(self, ids) -> np.ndarray:
        """Rows E[ids] of the [V, H] embedding, generated element-wise (no full table needed)."""
        H = self.m.hidden
        ids = np.asarray(ids, dtype=np.int64)
        out = np.empty((ids.shape[0], H), dtype=self.dtype)
        uniq, inv = np.unique(ids, return_inverse=True)
        rows = np.stack([gen(self.m.weight_seed, T_EMBED, H, scale_for("embed"), int(v) * H) for v in uniq]) \
            if len(uniq) else np.empty((0, H), np.float32)
        out[:] = rows[inv]
        return out

    def lm_head(self) -> np.ndarray:
        m = self.m
        return self._mat(T_LMHEAD, m.vocab, m.hidden, scale_for("proj", m.hidden))

    def final_norm(self) -> np.ndarray:
        return np.ones(self.m.hidden, self.dtype)
