"""ORACLE (test infrastructure only) -- plain fp32 decoder-only transformer forward.

What it computes (§2.1: a decoder-only LLM generating tokens
autoregressively; prefill computes the prompt's KV cache and the first output
token, decode one token per iteration, L58/L77-L79).  The layer is the
Llama / Qwen2 variant of the models the paper serves (L218, L224) [ext: HF
convention], in the order of SURVEY.md §8(c) O3:

    h = RMSNorm(x; g1)                        y = x / sqrt(mean(x^2) + eps) * g
    q, k, v = h Wq^T (+bq), h Wk^T (+bk), h Wv^T (+bv)
    q, k = RoPE(q, pos), RoPE(k, pos)         rotate-half pairs (i, i + d/2),
                                              inv_freq_i = theta^(-2i/d), angle = pos * inv_freq_i
    cache[slot(t)] = k, v                     (the oracle's own paged cache, O2)
    a = softmax(q K^T / sqrt(d)) V            keys 0..pos of the same sequence;
                                              GQA kv head = h // (Hq / Hkv)
    x += a Wo^T
    h = RMSNorm(x; g2)
    x += (silu(h Wg^T) * (h Wu^T)) Wd^T
  last stage: logits = RMSNorm(x; gf) Wlm^T, token = argmax (lowest id on ties, R18)

Two entry points:
  * `dense_forward`  -- the plain definition: one sequence, unbatched,
    unchunked, un-paged, full causal attention.
  * `stage_forward`  -- the same arithmetic over one scheduled mixed batch
    (chunked-prefill + decode tokens) with the oracle's own paged KV cache.
    Because paging, chunking and batching are exact reorderings, it must equal
    `dense_forward` row by row (tests/test_oracle_model.py).

Weights are the exact bf16 values of O4 held in fp32; KV and activations fp32
(north_star: "a plain fp32 CPU transformer forward"); `dtype=np.float64` is
available for pins.  Pinned by: HF `transformers` Llama/Qwen2 fp32 forward on
the same weights, fp64 brute-force attention, chunked == unchunked,
decode == full recompute, textbook RMSNorm / SiLU / RoPE closed forms.
"""
from __future__ import annotations

import numpy as np


def rmsnorm(x, g, eps):
    x = np.asarray(x)
    ms = np.mean(x * x, axis=-1, keepdims=True)
    return (x / np.sqrt(ms + x.dtype.type(eps))) * g


def silu(x):
    return x / (1.0 + np.exp(-x))


def rope(x, pos, theta):
    """x [T, nh, d], pos [T] -> rotated x (rotate-half convention)."""
    d = x.shape[-1]
    half = d // 2
    inv_freq = theta ** (-(2.0 * np.arange(half, dtype=np.float64)) / d)
    ang = np.asarray(pos, dtype=np.float64)[:, None] * inv_freq[None, :]     # [T, half]
    cos = np.cos(ang).astype(x.dtype)[:, None, :]
    sin = np.sin(ang).astype(x.dtype)[:, None, :]
    x1, x2 = x[..., :half], x[..., half:]
    return np.concatenate([x1 * cos - x2 * sin, x2 * cos + x1 * sin], axis=-1)


def attention(q, k, v, q_pos, k_pos):
    """q [Tq, Hq, d]; k, v [Tk, Hkv, d]; query t attends keys with k_pos <= q_pos[t]."""
    Hq, d = q.shape[1], q.shape[2]
    Hkv = k.shape[1]
    grp = Hq // Hkv
    kh = np.repeat(k, grp, axis=1)            # head h uses kv head h // grp
    vh = np.repeat(v, grp, axis=1)
    s = np.einsum("thd,shd->hts", q, kh) / q.dtype.type(np.sqrt(d))
    mask = np.asarray(k_pos)[None, :] <= np.asarray(q_pos)[:, None]          # [Tq, Tk]
    s = np.where(mask[None], s, -np.inf)
    s = s - s.max(axis=-1, keepdims=True)
    p = np.exp(s)
    p = p / p.sum(axis=-1, keepdims=True)
    return np.einsum("hts,shd->thd", p, vh)


def _qkv(m, w, h, pos):
    T = h.shape[0]
    q = h @ w["wq"].T
    k = h @ w["wk"].T
    v = h @ w["wv"].T
    if m.qkv_bias:
        q = q + w["bq"]
        k = k + w["bk"]
        v = v + w["bv"]
    q = rope(q.reshape(T, m.n_heads, m.head_dim), pos, m.rope_theta)
    k = rope(k.reshape(T, m.n_kv_heads, m.head_dim), pos, m.rope_theta)
    return q, k, v.reshape(T, m.n_kv_heads, m.head_dim)


def _mlp(m, w, x):
    h = rmsnorm(x, w["g2"], m.rms_eps)
    return x + (silu(h @ w["wg"].T) * (h @ w["wu"].T)) @ w["wd"].T


def dense_forward(m, W, ids, layers=None, x0=None):
    """Plain definition: hidden states [n_layers+1][T, H] of one sequence's prefix, and logits [T, V]."""
    ids = np.asarray(ids)
    T = ids.shape[0]
    pos = np.arange(T)
    x = W.embed_rows(ids) if x0 is None else np.array(x0, dtype=W.dtype)
    hs = [x]
    for l in (range(m.n_layers) if layers is None else layers):
        w = W.layer(l)
        h = rmsnorm(x, w["g1"], m.rms_eps)
        q, k, v = _qkv(m, w, h, pos)
        a = attention(q, k, v, pos, pos).reshape(T, m.q_dim)
        x = x + a @ w["wo"].T
        x = _mlp(m, w, x)
        hs.append(x)
    return hs


def logits_of(m, W, x):
    return rmsnorm(x, W.final_norm(), m.rms_eps) @ W.lm_head().T


def greedy(logits):
    """argmax with ties to the lowest id (R18): np.argmax returns the first maximum."""
    return np.argmax(logits, axis=-1).astype(np.int32)


class PagedCache:
    """The oracle's own paged KV cache: per layer, block id -> (K [bs, Hkv, d], V [bs, Hkv, d])."""

    def __init__(self, m, block_size, dtype=np.float32):
        self.m, self.bs, self.dtype = m, block_size, dtype
        self.k, self.v = {}, {}

    def write(self, layer, slots, k, v):
        K = self.k.setdefault(layer, {})
        V = self.v.setdefault(layer, {})
        shape = (self.bs, self.m.n_kv_heads, self.m.head_dim)
        for t, s in enumerate(np.asarray(slots)):
            b, o = divmod(int(s), self.bs)
            if b not in K:
                K[b] = np.zeros(shape, self.dtype)
                V[b] = np.zeros(shape, self.dtype)
            K[b][o] = k[t]
            V[b][o] = v[t]

    def fill_warm(self, layer, blocks, k, v):
        """Cached K/V of a warm sequence (O4 warm start): positions [0, len(k)) through its blocks."""
        n = k.shape[0]
        pos = np.arange(n)
        slots = np.asarray(blocks, np.int64)[pos // self.bs] * self.bs + pos % self.bs
        self.write(layer, slots, k.astype(self.dtype), v.astype(self.dtype))

    def gather(self, layer, blocks, n):
        """Keys/values of logical positions [0, n) through a block-table row."""
        K, V = self.k[layer], self.v[layer]
        nb = -(-n // self.bs)
        kk = np.concatenate([K[int(b)] for b in blocks[:nb]], axis=0)[:n]
        vv = np.concatenate([V[int(b)] for b in blocks[:nb]], axis=0)[:n]
        return kk, vv


def stage_forward(m, W, cache, batch, layer_begin, layer_end, hidden_in=None):
    """One pipeline stage over one mixed batch (oracle.scheduler.Batch or equivalent).

    Returns dict(hidden=[T, H] residual after layer_end-1, and on the last
    stage logits=[S_samp, V], sampled=[S_samp]).
    """
    T = batch.num_tokens
    pos = np.asarray(batch.positions)
    if layer_begin == 0:
        x = W.embed_rows(batch.token_ids)
    else:
        x = np.array(hidden_in, dtype=W.dtype, copy=True)
    cu = np.asarray(batch.cu_q)
    S = cu.shape[0] - 1
    for l in range(layer_begin, layer_end):
        w = W.layer(l)
        h = rmsnorm(x, w["g1"], m.rms_eps)
        q, k, v = _qkv(m, w, h, pos)
        cache.write(l, batch.slot_mapping, k, v)          # KV append before attention (causal within chunk)
        a = np.zeros((T, m.n_heads, m.head_dim), dtype=W.dtype)
        for i in range(S):
            t0, t1 = int(cu[i]), int(cu[i + 1])
            n = int(batch.kv_len[i])
            kk, vv = cache.gather(l, batch.block_table[i], n)
            a[t0:t1] = attention(q[t0:t1], kk, vv, pos[t0:t1], np.arange(n))
        x = x + a.reshape(T, m.q_dim) @ w["wo"].T
        x = _mlp(m, w, x)
    out = dict(hidden=x)
    if layer_end == m.n_layers:
        rows = x[np.asarray(batch.sample_idx, dtype=np.int64)]
        lg = logits_of(m, W, rows) if rows.shape[0] else np.zeros((0, m.vocab), W.dtype)
        out["logits"] = lg
        out["sampled"] = greedy(lg) if rows.shape[0] else np.zeros(0, np.int32)
    return out
